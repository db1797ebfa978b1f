// Microbenchmark (not product code): per-warp pane-table accumulation of
// (key, f32 value) pairs on sm_100a -- C3's shape (64 keys, values in [0,1)).
//   A: fp64 atomicAdd (a CAS loop on sm_100a) + u32 count atomicAdd
//   B: exact fixed point, 16-bit chunks of x*2^32 in two u32 limbs (red.shared.add,
//      no return value) + u32 count -- no CAS, no scoreboard wait
//   C: as B but the count rides in a third limb only every 8th update (not exact; bound)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubp scripts/ubench_pane_accum.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned hsh(unsigned x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
__device__ __forceinline__ void red_add(unsigned *p, unsigned v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(p)), "r"(v) : "memory");
}

template <int MODE, int G>
__global__ void __launch_bounds__(256) k(int iters, double *out) {
  __shared__ double fs[8 * G * 2];
  __shared__ unsigned cs[8 * G * 4];
  const int w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 8 * G * 2; i += 256) fs[i] = 0;
  for (int i = threadIdx.x; i < 8 * G * 4; i += 256) cs[i] = 0;
  __syncthreads();
  unsigned s = hsh(blockIdx.x * 256 + threadIdx.x);
  for (int it = 0; it < iters; ++it) {
    s = hsh(s + it);
    const int key = s % G;
    const float x = (float)(s >> 8) * (1.0f / 16777216.0f);
    if (MODE == 0) {
      atomicAdd(&fs[w * G + key], (double)x);
      atomicAdd(&cs[w * G + key], 1u);
    } else if (MODE == 1) {
      const unsigned V = (unsigned)(x * 4294967296.0f);   // exact for u24 values
      red_add(&cs[(w * 3 + 0) * G + key], 1u);
      red_add(&cs[(w * 3 + 1) * G + key], V & 0xffffu);
      red_add(&cs[(w * 3 + 2) * G + key], V >> 16);
    } else {
      const unsigned V = (unsigned)(x * 4294967296.0f);
      red_add(&cs[(w * 2 + 0) * G + key], (V & 0xffffu) | (1u << 16));   // low chunk + count? overflow bound only
      red_add(&cs[(w * 2 + 1) * G + key], V >> 16);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = fs[0] + cs[1];
}

template <int MODE, int G>
void run(const char *name) {
  double *out;
  cudaMalloc(&out, 148 * 8 * sizeof(double));
  int blocks = 148 * 4;
  int iters = 4096;
  k<MODE, G><<<blocks, 256>>>(16, out);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  k<MODE, G><<<blocks, 256>>>(iters, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double upd = (double)blocks * 256 * iters;
  printf("%-44s G=%5d  %.3f ns/update/GPU  %.2f SM-cycles/update  (err=%s)\n", name, G, ms * 1e6 / upd,
         ms * 1e-3 * 1.965e9 * 148 / upd, cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  run<0, 64>("A fp64 CAS atomic + u32 count");
  run<1, 64>("B 2 fixed-point limbs + count (red, 3 ops)");
  run<2, 64>("C 2 limbs, count folded (2 ops, bound)");
  run<0, 128>("A fp64 CAS atomic + u32 count");
  run<1, 128>("B 2 fixed-point limbs + count (red, 3 ops)");
  run<0, 16>("A fp64 CAS atomic + u32 count");
  run<1, 16>("B 2 fixed-point limbs + count (red, 3 ops)");
  return 0;
}
