// Microbenchmark (not product code): the read-only HBM ceiling a streaming scan
// can reach on this B200, to put k_pane_cnt's achieved GB/s in context (the
// MEASURED_PEAKS copy figure counts read + write bytes).
//   A: LDG.128 grid-stride, 4 loads in flight per thread, XOR-reduced (no stores)
//   B: 1-D TMA bulk copies into a 2-stage x 16 KiB shared ring per CTA, 4 CTAs/SM
//      (k_pane_cnt's staging geometry), each stage touched by one word per thread
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubr scripts/ubench_read_bw.cu && /tmp/ubr
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) k_ldg(const uint4 *__restrict__ p, size_t n16, unsigned *out) {
  unsigned acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    const uint4 a = __ldcs(p + i), b = __ldcs(p + i + stride), c = __ldcs(p + i + 2 * stride),
                d = __ldcs(p + i + 3 * stride);
    acc ^= a.x ^ b.y ^ c.z ^ d.w;
  }
  for (; i < n16; i += stride) acc ^= __ldcs(p + i).x;
  if (acc == 0x12345678u) out[0] = acc;
}

__device__ __forceinline__ uint32_t su(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int STAGES, int SB>
__global__ void __launch_bounds__(256) k_tma(const unsigned char *__restrict__ p, size_t n, unsigned *out) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t full[STAGES];
  const size_t per = ((n + gridDim.x - 1) / gridDim.x + SB - 1) / SB * SB;
  const size_t lo = (size_t)blockIdx.x * per, hi = lo + per < n ? lo + per : n;
  const int nst = hi > lo ? (int)((hi - lo + SB - 1) / SB) : 0;
  if (threadIdx.x == 0)
    for (int s = 0; s < STAGES; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(&full[s])));
  __syncthreads();
  auto issue = [&](int k) {
    const int s = k % STAGES;
    const size_t off = lo + (size_t)k * SB;
    const uint32_t bytes = (uint32_t)((hi - off) < SB ? (hi - off) : SB);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&full[s])), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su(sm + s * SB)), "l"(p + off), "r"(bytes), "r"(su(&full[s])) : "memory");
  };
  if (threadIdx.x == 0)
    for (int k = 0; k < STAGES && k < nst; ++k) issue(k);
  unsigned acc = 0;
  for (int k = 0; k < nst; ++k) {
    const int s = k % STAGES;
    const uint32_t ph = (k / STAGES) & 1;
    asm volatile("{\n .reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n @!P bra W;\n}\n" ::"r"(
                     su(&full[s])), "r"(ph) : "memory");
    acc ^= ((const unsigned *)(sm + s * SB))[threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0 && k + STAGES < nst) issue(k + STAGES);
  }
  if (acc == 0x12345678u) out[0] = acc;
}

int main() {
  const size_t n = 4ull << 30;
  unsigned char *d;
  unsigned *o;
  cudaMalloc(&d, n);
  cudaMalloc(&o, 4);
  cudaMemset(d, 1, n);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto time = [&](const char *name, auto launch) {
    float best = 1e30f;
    for (int r = 0; r < 10; ++r) {
      cudaEventRecord(a);
      launch();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (ms < best) best = ms;
    }
    printf("%-34s %8.3f ms  %7.1f GB/s\n", name, best, n / (best * 1e-3) / 1e9);
  };
  for (int bps : {4, 8, 16})
    time(bps == 4 ? "LDG.128 x4, 4 CTA/SM" : bps == 8 ? "LDG.128 x4, 8 CTA/SM" : "LDG.128 x4, 16 CTA/SM",
         [&] { k_ldg<<<sms * bps, 256>>>((const uint4 *)d, n / 16, o); });
  cudaFuncSetAttribute(k_tma<2, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 16384);
  cudaFuncSetAttribute(k_tma<3, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * 16384);
  cudaFuncSetAttribute(k_tma<4, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 16384);
  cudaFuncSetAttribute(k_tma<2, 32768>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 32768);
  time("TMA 2x16K ring, 4 CTA/SM", [&] { k_tma<2, 16384><<<sms * 4, 256, 2 * 16384>>>(d, n, o); });
  time("TMA 3x16K ring, 4 CTA/SM", [&] { k_tma<3, 16384><<<sms * 4, 256, 3 * 16384>>>(d, n, o); });
  time("TMA 4x16K ring, 3 CTA/SM", [&] { k_tma<4, 16384><<<sms * 3, 256, 4 * 16384>>>(d, n, o); });
  time("TMA 2x32K ring, 3 CTA/SM", [&] { k_tma<2, 32768><<<sms * 3, 256, 2 * 32768>>>(d, n, o); });
  time("copy (cudaMemcpy D2D, 2 GiB)", [&] { cudaMemcpyAsync(d, d + n / 2, n / 2, cudaMemcpyDeviceToDevice); });
  return 0;
}
