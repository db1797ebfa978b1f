// Microbenchmark (not product code): cost per update of shared-memory
// accumulation strategies on sm_100a, for the pane-aggregation design choice.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ub scripts/ubench_smem_atomics.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned hsh(unsigned x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

// MODE 0: smem atomicAdd(double)+atomicAdd(u32), per-warp table of G entries
// MODE 1: plain lane-private RMW (table [G][32])
// MODE 2: smem atomics on a CTA-shared table of G entries
template <int MODE, int G>
__global__ void __launch_bounds__(256) k(int iters, double *out) {
  constexpr int N = (MODE == 1) ? 8 * 32 * G : (MODE == 0 ? 8 * G : G);
  __shared__ double fs[N];
  __shared__ unsigned cs[N];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < N; i += 256) { fs[i] = 0; cs[i] = 0; }
  __syncthreads();
  unsigned s = hsh(blockIdx.x * 256 + threadIdx.x);
  for (int it = 0; it < iters; ++it) {
    s = hsh(s + it);
    const int key = s % G;
    const double v = (double)(s & 1023);
    if (MODE == 0) {
      atomicAdd(&fs[w * G + key], v);
      atomicAdd(&cs[w * G + key], 1u);
    } else if (MODE == 1) {
      fs[(w * G + key) * 32 + lane] += v;
      cs[(w * G + key) * 32 + lane] += 1u;
    } else {
      atomicAdd(&fs[key], v);
      atomicAdd(&cs[key], 1u);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = fs[0] + cs[1];
}

template <int MODE, int G>
void run(const char *name) {
  double *out;
  cudaMalloc(&out, 148 * 8 * sizeof(double));
  int blocks = 148 * 3;
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
  printf("%-34s G=%5d  %.3f ns/update/GPU  %.2f SM-cycles/update  (err=%s)\n", name, G, ms * 1e6 / upd,
         ms * 1e-3 * 1.965e9 * 148 / upd, cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  run<0, 64>("warp table, smem atomics");
  run<0, 4>("warp table, smem atomics");
  run<0, 1>("warp table, smem atomics");
  run<1, 4>("lane-private plain RMW");
  run<1, 1>("lane-private plain RMW");
  run<2, 64>("CTA table, smem atomics");
  run<2, 1024>("CTA table, smem atomics");
  return 0;
}
