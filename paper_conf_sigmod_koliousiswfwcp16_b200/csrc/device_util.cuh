// device_util.cuh -- small device helpers for the SABER hot path (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "plan.h"

namespace sb {

constexpr unsigned kFull = 0xffffffffu;
constexpr uint64_t kEmpty = ~0ull;          // empty hash slot

// Streaming 128-bit load that does not allocate in L1 (tuples are read once).
__device__ __forceinline__ uint4 ld_stream(const uint4 *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// Select word i of a register-resident tuple without local-memory indexing.
template <int NW>
__device__ __forceinline__ uint32_t sel_word(const uint32_t (&w)[NW], int i) {
  uint32_t r = w[0];
#pragma unroll
  for (int k = 1; k < NW; ++k) r = (i == k) ? w[k] : r;
  return r;
}

template <int NW>
__device__ __forceinline__ int64_t get_int(const uint32_t (&w)[NW], int word, int type) {
  uint32_t lo = sel_word<NW>(w, word);
  if (type == T_I32) return (int64_t)(int32_t)lo;
  uint32_t hi = sel_word<NW>(w, word + 1);
  return (int64_t)(((uint64_t)hi << 32) | lo);
}

template <int NW>
__device__ __forceinline__ double get_float(const uint32_t (&w)[NW], int word, int type) {
  uint32_t lo = sel_word<NW>(w, word);
  if (type == T_F32) return (double)__uint_as_float(lo);
  uint32_t hi = sel_word<NW>(w, word + 1);
  return __hiloint2double((int)hi, (int)lo);
}

template <class T>
__device__ __forceinline__ bool cmp_op(T a, int op, T b) {
  switch (op) {
    case OP_LT: return a < b;
    case OP_LE: return a <= b;
    case OP_GT: return a > b;
    case OP_GE: return a >= b;
    case OP_EQ: return a == b;
    default: return a != b;
  }
}

// order-preserving u64 encodings used by MIN/MAX fields
__device__ __forceinline__ uint64_t enc_int(int64_t v) { return (uint64_t)v ^ 0x8000000000000000ull; }
__device__ __forceinline__ int64_t dec_int(uint64_t u) { return (int64_t)(u ^ 0x8000000000000000ull); }
__device__ __forceinline__ uint64_t enc_dbl(double d) {
  uint64_t b = (uint64_t)__double_as_longlong(d);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__device__ __forceinline__ double dec_dbl(uint64_t u) {
  uint64_t b = (u >> 63) ? (u & 0x7fffffffffffffffull) : ~u;
  return __longlong_as_double((long long)b);
}

__device__ __forceinline__ uint64_t fmix64(uint64_t k) {
  k ^= k >> 33; k *= 0xff51afd7ed558ccdull;
  k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull;
  k ^= k >> 33;
  return k;
}

__device__ __forceinline__ uint64_t field_identity(int kind) {
  return kind == FK_MIN ? ~0ull : 0ull;
}

// combine two field values of the same kind
__device__ __forceinline__ uint64_t field_combine(int kind, uint64_t a, uint64_t b) {
  switch (kind) {
    case FK_SUM_F: return (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) +
                                                         __longlong_as_double((long long)b));
    case FK_SUM_I: return a + b;
    case FK_MIN: return a < b ? a : b;
    default: return a > b ? a : b;
  }
}

// field_combine without branches (op = FK_*; counts use FK_SUM_I), for loops
// whose field kind varies across the lanes of a warp
__device__ __forceinline__ uint64_t field_combine_sel(int op, uint64_t a, uint64_t b) {
  const uint64_t si = a + b;
  const uint64_t sf = (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) + __longlong_as_double((long long)b));
  const uint64_t mn = a < b ? a : b, mx = a < b ? b : a;
  return op == FK_SUM_F ? sf : op == FK_SUM_I ? si : op == FK_MIN ? mn : mx;
}

__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
  uint32_t lo = __shfl_sync(kFull, (uint32_t)v, src);
  uint32_t hi = __shfl_sync(kFull, (uint32_t)(v >> 32), src);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl_up64(uint64_t v, int d = 1) {
  const uint32_t lo = __shfl_up_sync(kFull, (uint32_t)v, d), hi = __shfl_up_sync(kFull, (uint32_t)(v >> 32), d);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl_down64(uint64_t v, int d) {
  const uint32_t lo = __shfl_down_sync(kFull, (uint32_t)v, d), hi = __shfl_down_sync(kFull, (uint32_t)(v >> 32), d);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl_xor64(uint64_t v, int m) {
  uint32_t lo = __shfl_xor_sync(kFull, (uint32_t)v, m);
  uint32_t hi = __shfl_xor_sync(kFull, (uint32_t)(v >> 32), m);
  return ((uint64_t)hi << 32) | lo;
}

__device__ __forceinline__ int64_t warp_min64(int64_t v) {
#pragma unroll
  for (int m = 16; m; m >>= 1) {
    int64_t o = (int64_t)shfl_xor64((uint64_t)v, m);
    v = o < v ? o : v;
  }
  return v;
}

// global atomics on pane-table words (return values unused → RED)
__device__ __forceinline__ void red_field(int kind, uint64_t *addr, uint64_t v) {
  switch (kind) {
    case FK_SUM_F: atomicAdd((double *)addr, __longlong_as_double((long long)v)); break;
    case FK_SUM_I: atomicAdd((unsigned long long *)addr, (unsigned long long)v); break;
    case FK_MIN: atomicMin((unsigned long long *)addr, (unsigned long long)v); break;
    default: atomicMax((unsigned long long *)addr, (unsigned long long)v); break;
  }
}

}  // namespace sb
