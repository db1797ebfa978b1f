// gen.cu -- device twin of saber_inputs/gen.py (counter-based stream generator).
// Input plumbing only: no windows, predicates or aggregates live here.  The
// bytes of tuple i depend only on (seed, i, params); a GPU test checks this
// kernel against the numpy generator byte for byte.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t r(uint64_t seed, uint64_t i, uint64_t c) {
  return splitmix64((seed << 48) ^ (i << 4) ^ c);
}
__device__ __forceinline__ float u24(uint64_t x) { return __fmul_rn((float)(x >> 40), 5.9604644775390625e-08f); }
__device__ __forceinline__ double u24d(uint64_t x) { return (double)(x >> 40) * 5.9604644775390625e-08; }
__device__ __forceinline__ int32_t u31(uint64_t x) { return (int32_t)(x >> 33); }
__device__ __forceinline__ int32_t uG(uint64_t x, uint64_t G) { return (int32_t)((x >> 32) % G); }

template <class T>
__device__ __forceinline__ void put(unsigned char *t, int off, T v) { *(T *)(t + off) = v; }

__global__ void k_gen(int kind, uint64_t seed, int64_t i0, int64_t n, int64_t rate, int64_t groups,
                      unsigned char *out) {
  const int tb = kind == 1 ? 64 : 32;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t i = (uint64_t)(i0 + k);
    unsigned char *t = out + k * tb;
    put<int64_t>(t, 0, (int64_t)(i / (uint64_t)rate));
    if (kind == 0) {  // Syn
      put<float>(t, 8, u24(r(seed, i, 1)));
      put<int32_t>(t, 12, uG(r(seed, i, 2), (uint64_t)groups));
      put<int32_t>(t, 16, u31(r(seed, i, 3)));
      put<int32_t>(t, 20, u31(r(seed, i, 4)));
      put<int32_t>(t, 24, u31(r(seed, i, 5)));
      put<int32_t>(t, 28, u31(r(seed, i, 6)));
    } else if (kind == 1) {  // CM
      put<int64_t>(t, 8, (int64_t)((r(seed, i, 1) >> 32) % 65536ull));
      put<int64_t>(t, 16, (int64_t)u31(r(seed, i, 2)));
      put<int64_t>(t, 24, (int64_t)u31(r(seed, i, 3)));
      put<int32_t>(t, 32, (int32_t)((r(seed, i, 4) >> 32) % 9ull));
      put<int32_t>(t, 36, u31(r(seed, i, 5)));
      put<int32_t>(t, 40, uG(r(seed, i, 6), (uint64_t)groups));
      put<int32_t>(t, 44, u31(r(seed, i, 7)));
      put<float>(t, 48, u24(r(seed, i, 8)));
      put<float>(t, 52, u24(r(seed, i, 9)));
      put<float>(t, 56, u24(r(seed, i, 10)));
      put<int32_t>(t, 60, u31(r(seed, i, 11)));
    } else if (kind == 2) {  // SG
      put<float>(t, 8, __fmul_rn(u24(r(seed, i, 1)), 1000.0f));
      put<int32_t>(t, 12, (int32_t)(r(seed, i, 2) & 1ull));
      const int32_t kk = uG(r(seed, i, 3), 2048);
      put<int32_t>(t, 16, kk & 7);
      put<int32_t>(t, 20, (kk >> 3) & 7);
      put<int32_t>(t, 24, kk >> 6);
      put<int32_t>(t, 28, 0);
    } else {  // LRB
      const int32_t hwy = uG(r(seed, i, 3), 8), lane = uG(r(seed, i, 4), 4), dir = uG(r(seed, i, 5), 2);
      const int32_t pos = (int32_t)((r(seed, i, 6) >> 32) % 528000ull);
      const int32_t seg = pos / 5280;
      const double base = ((hwy * 200 + dir * 100 + seg) % 4 == 0) ? 30.0 : 60.0;
      const double sp = __dadd_rn(__dsub_rn(base, 10.0), __dmul_rn(20.0, u24d(r(seed, i, 2))));
      put<int32_t>(t, 8, u31(r(seed, i, 1)) % (1 << 17));
      put<float>(t, 12, __double2float_rn(sp));
      put<int32_t>(t, 16, hwy);
      put<int32_t>(t, 20, lane);
      put<int32_t>(t, 24, dir);
      put<int32_t>(t, 28, pos);
    }
  }
}

}  // namespace

extern "C" int saber_gen(int kind, uint64_t seed, int64_t i0, int64_t n, int64_t rate, int64_t groups,
                         void *dev_out, void *stream) {
  if (n <= 0) return 0;
  int64_t blocks = (n + 255) / 256;
  if (blocks > 148 * 32) blocks = 148 * 32;
  k_gen<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(kind, seed, i0, n, rate, groups, (unsigned char *)dev_out);
  return (int)cudaGetLastError();
}

// Fill a device buffer (e.g. an L2 flush buffer) -- plumbing for the bench.
extern "C" int saber_gen_fill(void *dev, int64_t nbytes, int value, void *stream) {
  return (int)cudaMemsetAsync(dev, value, (size_t)nbytes, (cudaStream_t)stream);
}
