// join.cu -- windowed θ-join of two streams: the n-ary query
// task v = (f^q, B = <b1, b2>) of PAPER.md §3 L415-422 with the θ-join operator
// (§2.4), evaluated per window and emitted as RStream (L401-405).
//
// Window j of the join is W1_j ⋈θ W2_j with W_j = [j·l, j·l+s) on each stream
// (reading A26).  As in the paper (§5.4: "the number of
// tuples that match the join predicate is counted and the results are compressed
// in the global GPGPU memory, as for selection"), a task runs two passes over the
// pairs of its closed windows:
//   k_join_pairs<false>  one thread per row a of W1_j tests a against every b of
//                        W2_j, staged through shared memory in chunks (one CTA per
//                        (window, 256 rows)); counts matches per (window, a)
//   k_join_scan          exclusive scan of the counts (tiles + decoupled look-back)
//   k_join_pairs<true>   the same loops write π1(a) ++ π2(b) at offset + rank:
//                        pairs of a window in (a, b) order
//   k_join_hdr           window headers
// Windows that span tasks read the earlier tuples from a carry of each stream
// (the uncovered tail, < s tuples), so the virtual input of a task is
// [carry ++ batch] per stream.  Count windows only; τ is not read except for the
// header timestamp (reading A7: τ of S1's first tuple of the window).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/saber.h"
#include "common.cuh"

namespace sb {

constexpr int kJoinMaxPred = 64, kJoinMaxProj = 16;
constexpr int kJoinThreads = 256;
constexpr int kJoinChunk = 1024;          // W2 tuples staged per shared-memory chunk
constexpr int kJoinScanPer = 8, kJoinScanTile = kJoinThreads * kJoinScanPer;

struct JPred { int32_t w1, t1, op, w2, t2, pad; };     // S1 word w1 (type t1) op S2 word w2 (type t2)
struct JoinPlan {
  int32_t tb1, tb2, ts_word1, npred;
  int64_t s, l;
  JPred pred[kJoinMaxPred];
  int32_t nw1, nw2;                         // projected 32-bit words from S1 / S2
  int32_t pw1[2 * kJoinMaxProj], pw2[2 * kJoinMaxProj];
  int64_t rows_cap;
};
// virtual input of one stream: positions [cpos, tpos) in the carry, [tpos, ...) in the batch
struct JIn { const unsigned char *carry, *task; int64_t cpos, tpos; int32_t tb, pad; };

__device__ __forceinline__ const unsigned char *jtuple(const JIn &v, int64_t pos) {
  return pos < v.tpos ? v.carry + (pos - v.cpos) * v.tb : v.task + (pos - v.tpos) * v.tb;
}
__device__ __forceinline__ bool jcmp(const JPred &pr, const unsigned char *a, const unsigned char *b) {
  const bool fa = pr.t1 == T_F32 || pr.t1 == T_F64, fb = pr.t2 == T_F32 || pr.t2 == T_F64;
  auto geti = [](const unsigned char *t, int w, int ty) -> int64_t {
    return ty == T_I32 ? (int64_t) * (const int32_t *)(t + 4 * w) : *(const int64_t *)(t + 4 * w);
  };
  auto getf = [](const unsigned char *t, int w, int ty) -> double {
    return ty == T_F32 ? (double)*(const float *)(t + 4 * w) : *(const double *)(t + 4 * w);
  };
  if (fa || fb) {
    const double x = fa ? getf(a, pr.w1, pr.t1) : (double)geti(a, pr.w1, pr.t1);
    const double y = fb ? getf(b, pr.w2, pr.t2) : (double)geti(b, pr.w2, pr.t2);
    return cmp_op(x, pr.op, y);
  }
  return cmp_op(geti(a, pr.w1, pr.t1), pr.op, geti(b, pr.w2, pr.t2));
}

// one CTA per (window, block of 256 rows of W1): thread = row a; W2 staged in chunks
template <bool EMIT>
__global__ void __launch_bounds__(kJoinThreads)
k_join_pairs(const JoinPlan p, JIn v1, JIn v2, int64_t J0, int64_t *__restrict__ counts,
             const int64_t *__restrict__ offs, unsigned char *__restrict__ rows) {
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned char *sa = smem;                                   // [256][tb1]: this CTA's rows of W1
  unsigned char *sb = smem + (size_t)kJoinThreads * p.tb1;    // [kJoinChunk][tb2]: a chunk of W2
  const int64_t w = blockIdx.x;
  const int64_t j = J0 + w;
  const int a_loc = blockIdx.y * kJoinThreads + threadIdx.x;
  const bool act = a_loc < p.s;
  const int64_t base = j * p.l;
  // stage this CTA's W1 rows (16-byte words)
  {
    const int64_t left = p.s - (int64_t)blockIdx.y * kJoinThreads;
    const int nrow = (int)(left < kJoinThreads ? left : kJoinThreads);
    const int wpt = p.tb1 / 16;
    for (int x = threadIdx.x; x < nrow * wpt; x += kJoinThreads) {
      const int r = x / wpt, c = x - r * wpt;
      ((uint4 *)(sa + (size_t)r * p.tb1))[c] =
          ((const uint4 *)jtuple(v1, base + (int64_t)blockIdx.y * kJoinThreads + r))[c];
    }
  }
  const unsigned char *ta = sa + (size_t)threadIdx.x * p.tb1;
  int64_t cnt = 0;
  int64_t out = 0;
  if (EMIT && act) out = offs[w * p.s + a_loc];
  const int orow = 4 * (p.nw1 + p.nw2);
  for (int64_t c0 = 0; c0 < p.s; c0 += kJoinChunk) {
    const int nb = (int)((p.s - c0) < kJoinChunk ? (p.s - c0) : kJoinChunk);
    __syncthreads();
    const int wpt = p.tb2 / 16;
    for (int x = threadIdx.x; x < nb * wpt; x += kJoinThreads) {
      const int r = x / wpt, c = x - r * wpt;
      ((uint4 *)(sb + (size_t)r * p.tb2))[c] = ((const uint4 *)jtuple(v2, base + c0 + r))[c];
    }
    __syncthreads();
    if (!act) continue;
    for (int bi = 0; bi < nb; ++bi) {
      const unsigned char *tbp = sb + (size_t)bi * p.tb2;
      bool ok = true;
      for (int k = 0; k < p.npred && ok; ++k) ok = jcmp(p.pred[k], ta, tbp);
      if (!ok) continue;
      if (EMIT) {
        if (out < p.rows_cap) {
          uint32_t *dst = (uint32_t *)(rows + out * orow);
          for (int c = 0; c < p.nw1; ++c) dst[c] = ((const uint32_t *)ta)[p.pw1[c]];
          for (int c = 0; c < p.nw2; ++c) dst[p.nw1 + c] = ((const uint32_t *)tbp)[p.pw2[c]];
        }
        ++out;
      } else {
        ++cnt;
      }
    }
  }
  if (!EMIT && act) counts[w * p.s + a_loc] = cnt;
}

// Fast path: every θ term compares two int32 columns (JOIN_r over Syn) and there
// are at most kJoinFastTerms of them.  Row a's operands live in registers; the
// chunk of W2 is staged column-wise (one int32 array per term: every lane of a
// warp reads the same b, a broadcast); the comparison op per term is uniform.
constexpr int kJoinFastTerms = 8;
template <bool EMIT>
__global__ void __launch_bounds__(kJoinThreads)
k_join_pairs_i32(const JoinPlan p, JIn v1, JIn v2, int64_t J0, int64_t *__restrict__ counts,
                 const int64_t *__restrict__ offs, unsigned char *__restrict__ rows) {
  extern __shared__ __align__(16) unsigned char smem[];
  int32_t *col = (int32_t *)smem;                              // [npred][kJoinChunk]
  const int64_t w = blockIdx.x;
  const int64_t base = (J0 + w) * p.l;
  const int a_loc = blockIdx.y * kJoinThreads + threadIdx.x;
  const bool act = a_loc < p.s;
  const int np = p.npred;
  const unsigned char *ta = act ? jtuple(v1, base + a_loc) : nullptr;
  int32_t av[kJoinFastTerms];
  uint32_t om[kJoinFastTerms];                                 // outcome bits of op: lt | eq << 1 | gt << 2
#pragma unroll
  for (int k = 0; k < kJoinFastTerms; ++k) {
    av[k] = (act && k < np) ? *(const int32_t *)(ta + 4 * p.pred[k].w1) : 0;
    const int op = k < np ? p.pred[k].op : OP_EQ;
    om[k] = op == OP_LT ? 1u : op == OP_LE ? 3u : op == OP_GT ? 4u : op == OP_GE ? 6u : op == OP_EQ ? 2u : 5u;
  }
  auto term = [&](int k, int32_t b) -> uint32_t {          // a_k op b as one bit, branch-free
    const int32_t a = av[k];
    return (om[k] >> (a < b ? 0 : (a == b ? 1 : 2))) & 1u;
  };
  int64_t cnt = 0, out = 0;
  if (EMIT && act) out = offs[w * p.s + a_loc];
  const int orow = 4 * (p.nw1 + p.nw2);
  for (int64_t c0 = 0; c0 < p.s; c0 += kJoinChunk) {
    const int nb = (int)((p.s - c0) < kJoinChunk ? (p.s - c0) : kJoinChunk);
    __syncthreads();
    for (int x = threadIdx.x; x < nb; x += kJoinThreads) {
      const unsigned char *tb = jtuple(v2, base + c0 + x);
#pragma unroll
      for (int k = 0; k < kJoinFastTerms; ++k)
        if (k < np) col[k * kJoinChunk + x] = *(const int32_t *)(tb + 4 * p.pred[k].w2);
    }
    __syncthreads();
    if (!act) continue;
    if constexpr (!EMIT) {
      // count pass: independent iterations, unrolled so the broadcast shared loads overlap
#pragma unroll 8
      for (int bi = 0; bi < nb; ++bi) {
        uint32_t ok = 1u;
#pragma unroll
        for (int k = 0; k < kJoinFastTerms; ++k)
          if (k < np) ok &= term(k, col[k * kJoinChunk + bi]);
        cnt += ok;
      }
    } else {
#pragma unroll 4
    for (int bi = 0; bi < nb; ++bi) {
      uint32_t ok = 1u;
#pragma unroll
      for (int k = 0; k < kJoinFastTerms; ++k)
        if (k < np) ok &= term(k, col[k * kJoinChunk + bi]);
      if (ok) {
        if (out < p.rows_cap) {
          const unsigned char *tb = jtuple(v2, base + c0 + bi);
          uint32_t *dst = (uint32_t *)(rows + out * orow);
          for (int c = 0; c < p.nw1; ++c) dst[c] = ((const uint32_t *)ta)[p.pw1[c]];
          for (int c = 0; c < p.nw2; ++c) dst[p.nw1 + c] = ((const uint32_t *)tb)[p.pw2[c]];
        }
        ++out;
      }
    }
    }
  }
  if (!EMIT && act) counts[w * p.s + a_loc] = cnt;
}


// Emission of the fast path with coalesced rows: a warp per row a of W1, lanes over
// the b's of the staged W2 chunk.  Row a's pairs are contiguous in the output, in b
// order, so a ballot over 32 consecutive b's places a lane's row at a's running
// offset + the popcount of the lower lanes: the warp writes 32 consecutive rows per
// step (the thread-per-row pass scattered every store over 32 rows far apart).  The
// θ columns and the projected words of the chunk are staged column-wise; lane l
// keeps the running offset of the warp's l-th row.  Same rows, same order as the
// thread-per-row kernel (pairs in (a, b) order, reading A26).
constexpr int kJoinEmitWords = 8;           // projected words of S2 staged per chunk
__global__ void __launch_bounds__(kJoinThreads)
k_join_emit_i32(const JoinPlan p, JIn v1, JIn v2, int64_t J0, const int64_t *__restrict__ offs,
                unsigned char *__restrict__ rows) {
  extern __shared__ __align__(16) unsigned char smem[];
  int32_t *col = (int32_t *)smem;                              // [npred][kJoinChunk]
  uint32_t *pj = (uint32_t *)(col + kJoinFastTerms * kJoinChunk);   // [nw2][kJoinChunk]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t w = blockIdx.x;
  const int64_t base = (J0 + w) * p.l;
  const int a0 = blockIdx.y * kJoinThreads;
  const int np = p.npred, nw1 = p.nw1, nw2 = p.nw2;
  const int orow = 4 * (nw1 + nw2);
  const unsigned lt = (1u << lane) - 1u;
  uint32_t om[kJoinFastTerms];
#pragma unroll
  for (int k = 0; k < kJoinFastTerms; ++k) {
    const int op = k < np ? p.pred[k].op : OP_EQ;
    om[k] = op == OP_LT ? 1u : op == OP_LE ? 3u : op == OP_GT ? 4u : op == OP_GE ? 6u : op == OP_EQ ? 2u : 5u;
  }
  // lane l: running output row, θ operands and projected words of a = a0 + warp + 8·l (held in
  // registers and broadcast by shuffles: no dependent global load per row)
  const int al = a0 + warp + 8 * lane;
  const bool lv = lane < kJoinThreads / 8 && al < p.s;
  int64_t run = lv ? offs[w * p.s + al] : 0;
  int32_t avl[kJoinFastTerms];
  uint32_t pwl[kJoinEmitWords];
  {
    const unsigned char *tal = lv ? jtuple(v1, base + al) : nullptr;
#pragma unroll
    for (int k = 0; k < kJoinFastTerms; ++k) avl[k] = (lv && k < np) ? *(const int32_t *)(tal + 4 * p.pred[k].w1) : 0;
#pragma unroll
    for (int c = 0; c < kJoinEmitWords; ++c) pwl[c] = (lv && c < nw1) ? ((const uint32_t *)tal)[p.pw1[c]] : 0u;
  }
  for (int64_t c0 = 0; c0 < p.s; c0 += kJoinChunk) {
    const int nb = (int)((p.s - c0) < kJoinChunk ? (p.s - c0) : kJoinChunk);
    __syncthreads();
    for (int x = tid; x < nb; x += kJoinThreads) {
      const unsigned char *tb = jtuple(v2, base + c0 + x);
#pragma unroll
      for (int k = 0; k < kJoinFastTerms; ++k)
        if (k < np) col[k * kJoinChunk + x] = *(const int32_t *)(tb + 4 * p.pred[k].w2);
#pragma unroll
      for (int c = 0; c < kJoinEmitWords; ++c)
        if (c < nw2) pj[c * kJoinChunk + x] = ((const uint32_t *)tb)[p.pw2[c]];
    }
    __syncthreads();
    for (int i = 0; i < kJoinThreads / 8; ++i) {
      const int a = a0 + warp + 8 * i;
      if (a >= p.s) break;                                     // warp-uniform
      int32_t av[kJoinFastTerms];
#pragma unroll
      for (int k = 0; k < kJoinFastTerms; ++k) av[k] = __shfl_sync(kFull, avl[k], i);
      uint32_t pa[kJoinEmitWords];
#pragma unroll
      for (int c = 0; c < kJoinEmitWords; ++c) pa[c] = __shfl_sync(kFull, pwl[c], i);
      int64_t out = (int64_t)__shfl_sync(kFull, (unsigned long long)run, i);
      for (int b0 = 0; b0 < nb; b0 += 32) {
        const int b = b0 + lane;
        uint32_t ok = b < nb ? 1u : 0u;
#pragma unroll
        for (int k = 0; k < kJoinFastTerms; ++k)
          if (k < np) {
            const int32_t y = col[k * kJoinChunk + (b < nb ? b : 0)];
            ok &= (om[k] >> (av[k] < y ? 0 : (av[k] == y ? 1 : 2))) & 1u;
          }
        const unsigned bal = __ballot_sync(kFull, ok);
        if (ok) {
          const int64_t r = out + __popc(bal & lt);
          if (r < p.rows_cap) {
            uint32_t *dst = (uint32_t *)(rows + r * orow);
#pragma unroll
            for (int c = 0; c < kJoinEmitWords; ++c)
              if (c < nw1) dst[c] = pa[c];
#pragma unroll
            for (int c = 0; c < kJoinEmitWords; ++c)
              if (c < nw2) dst[nw1 + c] = pj[c * kJoinChunk + b];
          }
        }
        out += __popc(bal);
      }
      if (lane == i) run = out;
    }
  }
}

// exclusive scan of n counts in place (tiles by ticket, decoupled look-back); the
// total goes to *total
__global__ void __launch_bounds__(kJoinThreads)
k_join_scan(int64_t *__restrict__ v, int64_t n, uint64_t *__restrict__ status, int *__restrict__ ticket,
            uint64_t epoch, int64_t *__restrict__ total) {
  __shared__ int64_t wsum[kJoinThreads / 32];
  __shared__ int64_t s_base;
  __shared__ int s_t;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t ntiles = (n + kJoinScanTile - 1) / kJoinScanTile;
  for (;;) {
    if (tid == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= ntiles) break;
    const int64_t a = t * kJoinScanTile + (int64_t)tid * kJoinScanPer;
    int64_t x[kJoinScanPer], loc = 0;
#pragma unroll
    for (int k = 0; k < kJoinScanPer; ++k) {
      x[k] = a + k < n ? v[a + k] : 0;
      loc += x[k];
    }
    int64_t y = loc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t z = (int64_t)__shfl_up_sync(kFull, (unsigned long long)y, o);
      if (lane >= o) y += z;
    }
    if (lane == 31) wsum[wid] = y;
    __syncthreads();
    if (wid == 0) {
      const int64_t ws = lane < kJoinThreads / 32 ? wsum[lane] : 0;
      int64_t u = ws;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t z = (int64_t)__shfl_up_sync(kFull, (unsigned long long)u, o);
        if (lane >= o) u += z;
      }
      if (lane < kJoinThreads / 32) wsum[lane] = u - ws;
      const uint64_t tt = (uint64_t)__shfl_sync(kFull, (unsigned long long)u, 31);
      const int64_t excl = lookback_warp(status, t, epoch, tt);
      if (lane == 0) {
        s_base = excl;
        if (t == ntiles - 1) *total = excl + (int64_t)tt;
      }
    }
    __syncthreads();
    int64_t run = s_base + wsum[wid] + y - loc;
#pragma unroll
    for (int k = 0; k < kJoinScanPer; ++k) {
      if (a + k < n) v[a + k] = run;
      run += x[k];
    }
    __syncthreads();
  }
}

__global__ void k_join_hdr(const JoinPlan p, JIn v1, int64_t J0, int64_t nwin, const int64_t *__restrict__ offs,
                           const int64_t *__restrict__ total, WinHdr *__restrict__ hdr) {
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nwin; w += (int64_t)gridDim.x * blockDim.x) {
    const int64_t o = offs[w * p.s], e = w + 1 < nwin ? offs[(w + 1) * p.s] : *total;
    WinHdr h;
    h.window_id = J0 + w;
    h.ts = *(const int64_t *)(jtuple(v1, (J0 + w) * p.l) + 4 * p.ts_word1);
    h.row_offset = o;
    h.nrows = (int32_t)(e - o);
    h.flags = 0;
    hdr[w] = h;
  }
}

}  // namespace sb

using namespace sb;

namespace {
thread_local std::string g_join_error;
int jtype_bytes(int t) { return (t == T_I32 || t == T_F32) ? 4 : 8; }

struct JSlot {
  unsigned char *rows = nullptr, *h_rows = nullptr;
  void *hdr = nullptr;
  saber_win_hdr *h_hdr = nullptr;
  int64_t *d_total = nullptr, *h_total = nullptr;
  cudaEvent_t done = nullptr;
  int64_t task_id = -1, first_window = 0, nwindows = 0;
  int state = 0;                   // 0 free, 1 busy, 2 polled
};
}  // namespace

struct saber_join {
  JoinPlan p{};
  saber_config cfg{};
  int device = 0;
  cudaStream_t cs = nullptr;
  int64_t task_tuples = 0, win_cap = 0;
  unsigned char *carry[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};   // [stream][buffer]
  int cur = 0;                     // carry buffer holding positions [cpos, tpos)
  unsigned char *stage[2] = {nullptr, nullptr};   // device copies of host batches
  int64_t cpos = 0, tpos = 0, J0 = 0;
  int64_t *counts = nullptr;
  uint64_t *status = nullptr;
  int64_t status_cap = 0;
  int *ticket = nullptr;
  uint64_t epoch = 0;
  std::vector<JSlot> slots;
  int64_t next_task = 0, next_poll = 0;
  bool fast = false;               // every θ term compares two int32 columns, <= kJoinFastTerms terms
  std::string err;
};

static saber_status jfail(saber_join *j, saber_status s, const std::string &m) {
  if (j) j->err = m;
  g_join_error = m;
  return s;
}
#define JCK(call)                                                                                \
  do {                                                                                           \
    cudaError_t e_ = (call);                                                                     \
    if (e_ != cudaSuccess) return jfail(j, SABER_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

static saber_status join_task(saber_join *j, const unsigned char *d1, const unsigned char *d2, int64_t n) {
  const JoinPlan &p = j->p;
  JSlot &s = j->slots[j->next_task % (int64_t)j->slots.size()];
  if (s.state != 0) return jfail(j, SABER_EAGAIN, "result slot busy: poll and release first");
  const int64_t total = j->tpos + n;
  const int64_t J1 = total >= p.s ? (total - p.s) / p.l + 1 : j->J0;
  const int64_t nwin = std::max<int64_t>(0, J1 - j->J0);
  if (nwin > j->win_cap) return jfail(j, SABER_EINVAL, "task closes more windows than a result slot holds");
  JIn v1{j->carry[0][j->cur], d1, j->cpos, j->tpos, p.tb1, 0};
  JIn v2{j->carry[1][j->cur], d2, j->cpos, j->tpos, p.tb2, 0};
  const size_t smem = (size_t)kJoinThreads * p.tb1 + (size_t)kJoinChunk * p.tb2;
  const bool fast = j->fast;
  const size_t fsmem = (size_t)kJoinFastTerms * kJoinChunk * 4;
  if (nwin > 0) {
    const dim3 grid((unsigned)nwin, (unsigned)((p.s + kJoinThreads - 1) / kJoinThreads));
    if (fast) k_join_pairs_i32<false><<<grid, kJoinThreads, fsmem, j->cs>>>(p, v1, v2, j->J0, j->counts, nullptr, nullptr);
    else k_join_pairs<false><<<grid, kJoinThreads, smem, j->cs>>>(p, v1, v2, j->J0, j->counts, nullptr, nullptr);
    JCK(cudaGetLastError());
    JCK(cudaMemsetAsync(j->ticket, 0, sizeof(int), j->cs));
    ++j->epoch;
    if ((j->epoch & 0xffffff) == 0) JCK(cudaMemsetAsync(j->status, 0, (size_t)j->status_cap * 8, j->cs));
    k_join_scan<<<148 * 4, kJoinThreads, 0, j->cs>>>(j->counts, nwin * p.s, j->status, j->ticket, j->epoch,
                                                     s.d_total);
    JCK(cudaGetLastError());
    if (fast && p.nw2 <= kJoinEmitWords && p.nw1 <= kJoinEmitWords && !std::getenv("SABER_JOIN_THREAD_EMIT"))
      k_join_emit_i32<<<grid, kJoinThreads, fsmem + (size_t)kJoinEmitWords * kJoinChunk * 4, j->cs>>>(
          p, v1, v2, j->J0, j->counts, s.rows);
    else if (fast) k_join_pairs_i32<true><<<grid, kJoinThreads, fsmem, j->cs>>>(p, v1, v2, j->J0, nullptr, j->counts, s.rows);
    else k_join_pairs<true><<<grid, kJoinThreads, smem, j->cs>>>(p, v1, v2, j->J0, nullptr, j->counts, s.rows);
    JCK(cudaGetLastError());
    k_join_hdr<<<148, 256, 0, j->cs>>>(p, v1, j->J0, nwin, j->counts, s.d_total, (WinHdr *)s.hdr);
    JCK(cudaGetLastError());
  } else {
    JCK(cudaMemsetAsync(s.d_total, 0, 8, j->cs));
  }
  // new carry: positions [max(J1·l, cpos), total) of the virtual input, into the other buffer
  const int64_t ncp = std::max(J1 * p.l, j->cpos);
  const int nb = j->cur ^ 1;
  for (int k = 0; k < 2; ++k) {
    const int tb = k == 0 ? p.tb1 : p.tb2;
    const unsigned char *task = k == 0 ? d1 : d2;
    int64_t at = ncp;
    unsigned char *dst = j->carry[k][nb];
    if (at < j->tpos) {
      const int64_t m = j->tpos - at;
      JCK(cudaMemcpyAsync(dst, j->carry[k][j->cur] + (at - j->cpos) * tb, (size_t)(m * tb), cudaMemcpyDeviceToDevice, j->cs));
      dst += m * tb;
      at = j->tpos;
    }
    if (total > at) JCK(cudaMemcpyAsync(dst, task + (at - j->tpos) * tb, (size_t)((total - at) * tb), cudaMemcpyDeviceToDevice, j->cs));
  }
  JCK(cudaMemcpyAsync(s.h_total, s.d_total, 8, cudaMemcpyDeviceToHost, j->cs));
  JCK(cudaEventRecord(s.done, j->cs));
  s.state = 1;
  s.task_id = j->next_task++;
  s.first_window = j->J0;
  s.nwindows = nwin;
  j->cur = nb;
  j->cpos = ncp;
  j->tpos = total;
  j->J0 = std::max(j->J0, J1);
  return SABER_OK;
}

extern "C" {

saber_status saber_join_create(const saber_schema *s1, const saber_schema *s2, const saber_join_op *op,
                               const saber_window *w, const saber_config *cfg, saber_join **out) {
  if (!out) return jfail(nullptr, SABER_EINVAL, "out is NULL");
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
    cudaGetLastError();
    return jfail(nullptr, SABER_ECUDA, "no CUDA device (there is no CPU path)");
  }
  if (!s1 || !s2 || !op || !w) return jfail(nullptr, SABER_EINVAL, "null argument");
  if (w->kind != SABER_WIN_COUNT) return jfail(nullptr, SABER_EINVAL, "θ-join: count windows only");
  if (w->size < 1 || w->slide < 1 || w->slide > w->size) return jfail(nullptr, SABER_EINVAL, "window");
  if (op->npred < 0 || op->npred > kJoinMaxPred || (op->npred && !op->theta)) return jfail(nullptr, SABER_EINVAL, "theta");
  if (op->nproj1 < 0 || op->nproj2 < 0 || op->nproj1 > kJoinMaxProj || op->nproj2 > kJoinMaxProj ||
      op->nproj1 + op->nproj2 < 1)
    return jfail(nullptr, SABER_EINVAL, "projection");
  saber_join *j = new saber_join();
  JoinPlan &p = j->p;
  auto schema_ok = [](const saber_schema *sc) {
    if (sc->tuple_bytes % 16 || sc->tuple_bytes < 16 || sc->tuple_bytes > 64 || sc->ncols < 1) return false;
    for (int c = 0; c < sc->ncols; ++c) {
      const int b = jtype_bytes(sc->types[c]);
      if (sc->types[c] < 0 || sc->types[c] > 3 || sc->offsets[c] % b || sc->offsets[c] + b > sc->tuple_bytes) return false;
    }
    return sc->ts_col >= 0 && sc->ts_col < sc->ncols && sc->types[sc->ts_col] == SABER_I64;
  };
  if (!schema_ok(s1) || !schema_ok(s2)) { delete j; return jfail(nullptr, SABER_EINVAL, "schema"); }
  p.tb1 = s1->tuple_bytes;
  p.tb2 = s2->tuple_bytes;
  p.ts_word1 = s1->offsets[s1->ts_col] / 4;
  p.s = w->size;
  p.l = w->slide;
  p.npred = op->npred;
  for (int k = 0; k < op->npred; ++k) {
    const saber_join_pred &pr = op->theta[k];
    if (pr.col1 < 0 || pr.col1 >= s1->ncols || pr.col2 < 0 || pr.col2 >= s2->ncols || pr.op < SABER_LT ||
        pr.op > SABER_NE) {
      delete j;
      return jfail(nullptr, SABER_EINVAL, "bad θ term");
    }
    p.pred[k] = JPred{s1->offsets[pr.col1] / 4, s1->types[pr.col1], pr.op, s2->offsets[pr.col2] / 4,
                      s2->types[pr.col2], 0};
  }
  auto proj = [&](const saber_schema *sc, int n, const int32_t *cols, int32_t *pw, int32_t &nw) {
    nw = 0;
    for (int c = 0; c < n; ++c) {
      if (cols[c] < 0 || cols[c] >= sc->ncols) return false;
      for (int k = 0; k < jtype_bytes(sc->types[cols[c]]) / 4; ++k) pw[nw++] = sc->offsets[cols[c]] / 4 + k;
    }
    return true;
  };
  if (!proj(s1, op->nproj1, op->proj1, p.pw1, p.nw1) || !proj(s2, op->nproj2, op->proj2, p.pw2, p.nw2)) {
    delete j;
    return jfail(nullptr, SABER_EINVAL, "bad projection column");
  }
  j->fast = op->npred <= kJoinFastTerms && !std::getenv("SABER_JOIN_GENERIC");
  for (int k = 0; k < op->npred; ++k) j->fast &= p.pred[k].t1 == T_I32 && p.pred[k].t2 == T_I32;
  if (cfg) j->cfg = *cfg;
  if (j->cfg.task_bytes <= 0) j->cfg.task_bytes = 32ll << 20;
  j->device = (cfg && cfg->device >= 0) ? cfg->device : 0;
  if (!cfg) cudaGetDevice(&j->device);
  j->task_tuples = j->cfg.task_bytes / p.tb1;
  j->win_cap = j->task_tuples / p.l + 4;
  const int64_t row_bytes = 4 * (p.nw1 + p.nw2);
  int64_t rb = j->cfg.result_bytes > 0 ? j->cfg.result_bytes : (256ll << 20);
  p.rows_cap = rb / row_bytes;
  const int nslots = j->cfg.result_slots > 0 ? j->cfg.result_slots : 4;
  j->slots.resize(nslots);
  auto setup = [&]() -> saber_status {
    JCK(cudaSetDevice(j->device));
    JCK(cudaStreamCreateWithFlags(&j->cs, cudaStreamNonBlocking));
    const int64_t cap = p.s + p.l + 16;
    for (int k = 0; k < 2; ++k)
      for (int b = 0; b < 2; ++b) JCK(cudaMalloc(&j->carry[k][b], (size_t)cap * (k == 0 ? p.tb1 : p.tb2)));
    JCK(cudaMalloc(&j->stage[0], (size_t)j->task_tuples * p.tb1));
    JCK(cudaMalloc(&j->stage[1], (size_t)j->task_tuples * p.tb2));
    JCK(cudaMalloc(&j->counts, (size_t)j->win_cap * p.s * 8));
    j->status_cap = (j->win_cap * p.s) / kJoinScanTile + 16;
    JCK(cudaMalloc(&j->status, (size_t)j->status_cap * 8));
    JCK(cudaMemset(j->status, 0, (size_t)j->status_cap * 8));
    JCK(cudaMalloc(&j->ticket, 64));
    for (auto &s : j->slots) {
      JCK(cudaMalloc(&s.rows, (size_t)p.rows_cap * row_bytes));
      JCK(cudaMalloc(&s.hdr, (size_t)j->win_cap * sizeof(saber_win_hdr)));
      JCK(cudaMalloc(&s.d_total, 8));
      JCK(cudaMallocHost(&s.h_total, 8));
      JCK(cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming));
      if (j->cfg.result_mode == SABER_RESULTS_HOST) {
        JCK(cudaMallocHost(&s.h_rows, (size_t)p.rows_cap * row_bytes));
        JCK(cudaMallocHost(&s.h_hdr, (size_t)j->win_cap * sizeof(saber_win_hdr)));
      }
    }
    const size_t smem = (size_t)kJoinThreads * p.tb1 + (size_t)kJoinChunk * p.tb2;
    JCK(cudaFuncSetAttribute((void *)k_join_pairs<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    JCK(cudaFuncSetAttribute((void *)k_join_pairs<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    JCK(cudaFuncSetAttribute((void *)k_join_emit_i32, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)((kJoinFastTerms + kJoinEmitWords) * kJoinChunk * 4)));
    return SABER_OK;
  };
  if (saber_status st = setup()) {
    saber_join_destroy(j);
    return st;
  }
  *out = j;
  return SABER_OK;
}

saber_status saber_join_submit_device(saber_join *j, const void *dev1, const void *dev2, size_t ntuples,
                                      void *cuda_stream) {
  if (!j) return jfail(nullptr, SABER_EINVAL, "null join");
  if ((int64_t)ntuples > j->task_tuples) return jfail(j, SABER_EINVAL, "batch larger than task_bytes");
  if (ntuples == 0) return SABER_OK;
  JCK(cudaSetDevice(j->device));
  cudaEvent_t ev;
  JCK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  JCK(cudaEventRecord(ev, (cudaStream_t)cuda_stream));
  JCK(cudaStreamWaitEvent(j->cs, ev, 0));
  saber_status st = join_task(j, (const unsigned char *)dev1, (const unsigned char *)dev2, (int64_t)ntuples);
  if (st == SABER_OK) {
    JCK(cudaEventRecord(ev, j->cs));
    JCK(cudaStreamWaitEvent((cudaStream_t)cuda_stream, ev, 0));
  }
  cudaEventDestroy(ev);
  return st;
}

saber_status saber_join_submit(saber_join *j, const void *host1, const void *host2, size_t ntuples) {
  if (!j) return jfail(nullptr, SABER_EINVAL, "null join");
  if ((int64_t)ntuples > j->task_tuples) return jfail(j, SABER_EINVAL, "batch larger than task_bytes");
  if (ntuples == 0) return SABER_OK;
  JSlot &s = j->slots[j->next_task % (int64_t)j->slots.size()];
  if (s.state != 0) return jfail(j, SABER_EAGAIN, "result slot busy: poll and release first");
  JCK(cudaSetDevice(j->device));
  JCK(cudaMemcpyAsync(j->stage[0], host1, ntuples * j->p.tb1, cudaMemcpyHostToDevice, j->cs));
  JCK(cudaMemcpyAsync(j->stage[1], host2, ntuples * j->p.tb2, cudaMemcpyHostToDevice, j->cs));
  saber_status st = join_task(j, j->stage[0], j->stage[1], (int64_t)ntuples);
  if (st == SABER_OK) JCK(cudaStreamSynchronize(j->cs));   // the staging buffers are reused by the next batch
  return st;
}

saber_status saber_join_poll(saber_join *j, saber_results *out, int32_t timeout_us) {
  if (!j || !out) return jfail(j, SABER_EINVAL, "poll arguments");
  std::memset(out, 0, sizeof(*out));
  if (j->next_poll >= j->next_task) return jfail(j, SABER_EAGAIN, "no pending task");
  JSlot &s = j->slots[j->next_poll % (int64_t)j->slots.size()];
  JCK(cudaSetDevice(j->device));
  if (timeout_us >= 0) {
    cudaError_t e = cudaEventQuery(s.done);
    if (e == cudaErrorNotReady && timeout_us == 0) { cudaGetLastError(); return jfail(j, SABER_EAGAIN, "not ready"); }
  }
  JCK(cudaEventSynchronize(s.done));
  const int64_t rows = *s.h_total;
  if (rows > j->p.rows_cap) return jfail(j, SABER_ENOMEM, "join result exceeds the result slot (raise result_bytes)");
  const int32_t rb = 4 * (j->p.nw1 + j->p.nw2);
  const bool host = j->cfg.result_mode == SABER_RESULTS_HOST;
  if (host) {
    if (rows) JCK(cudaMemcpy(s.h_rows, s.rows, (size_t)rows * rb, cudaMemcpyDeviceToHost));
    if (s.nwindows) JCK(cudaMemcpy(s.h_hdr, s.hdr, (size_t)s.nwindows * sizeof(saber_win_hdr), cudaMemcpyDeviceToHost));
  }
  out->task_id = s.task_id;
  out->first_window = s.first_window;
  out->nwindows = s.nwindows;
  out->hdr = host ? s.h_hdr : (const saber_win_hdr *)s.hdr;
  out->on_device = !host;
  out->tuples = host ? (const void *)s.h_rows : (const void *)s.rows;
  out->tuple_bytes = rb;
  out->ntuples = rows;
  s.state = 2;
  j->next_poll++;
  return SABER_OK;
}

saber_status saber_join_release(saber_join *j, const saber_results *r) {
  if (!j || !r) return jfail(j, SABER_EINVAL, "release arguments");
  JSlot &s = j->slots[r->task_id % (int64_t)j->slots.size()];
  if (s.task_id != r->task_id || s.state != 2) return jfail(j, SABER_EINVAL, "slice not polled or released twice");
  s.state = 0;
  return SABER_OK;
}

void saber_join_destroy(saber_join *j) {
  if (!j) return;
  cudaSetDevice(j->device);
  if (j->cs) cudaStreamSynchronize(j->cs);
  for (auto &s : j->slots) {
    cudaFree(s.rows); cudaFree(s.hdr); cudaFree(s.d_total);
    cudaFreeHost(s.h_total); cudaFreeHost(s.h_rows); cudaFreeHost(s.h_hdr);
    if (s.done) cudaEventDestroy(s.done);
  }
  for (int k = 0; k < 2; ++k) {
    cudaFree(j->stage[k]);
    for (int b = 0; b < 2; ++b) cudaFree(j->carry[k][b]);
  }
  cudaFree(j->counts); cudaFree(j->status); cudaFree(j->ticket);
  if (j->cs) cudaStreamDestroy(j->cs);
  cudaGetLastError();
  delete j;
}

const char *saber_join_last_error(const saber_join *j) { return j ? j->err.c_str() : g_join_error.c_str(); }

}  // extern "C"
