// atomics_bench.cu — B200 primitive rates that bound the GROUP BY paths (DESIGN.md §Measured
// constants). Standalone: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ab atomics_bench.cu
//   1. random 8-byte loads (one sector each) over a table of T bytes            -> probe rate
//   2. random REDG.ADD.64 over T bytes (1 and 3 fields per 32-byte slot)        -> slot-update rate
//   3. shared-memory ATOMS.ADD.32 / 64-bit CAS-loop add / f64 add over D entries -> path (a) rate
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t h) {
  h ^= h >> 33; h *= 0xff51afd7ed558ccdull; h ^= h >> 33; h *= 0xc4ceb9fe1a85ec53ull; h ^= h >> 33; return h;
}

__global__ void k_rand_load(const uint64_t* t, uint64_t mask, uint64_t n, uint64_t* sink) {
  uint64_t acc = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t s = mix(i) & mask;
    acc += __ldcg(t + s * 4);  // 32-byte slots
  }
  if (acc == 42) *sink = acc;
}

template <int F>
__global__ void k_rand_red(uint64_t* t, uint64_t mask, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t s = mix(i) & mask;
#pragma unroll
    for (int f = 0; f < F; ++f) atomicAdd((unsigned long long*)(t + s * 4 + 1 + f), 1ull);
  }
}

template <int MODE>
__global__ void k_smem(uint64_t n, uint32_t D, uint64_t* out) {
  extern __shared__ uint64_t sm[];
  for (uint32_t e = threadIdx.x; e < D; e += blockDim.x) sm[e] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t e = (uint32_t)(mix(i) % D);
    if (MODE == 0) atomicAdd((uint32_t*)sm + e, 1u);
    if (MODE == 1) atomicAdd((unsigned long long*)sm + e, 3ull);
    if (MODE == 2) atomicAdd((double*)sm + e, 1.5);
    if (MODE == 3) { uint32_t old = atomicAdd((uint32_t*)sm + e, 7u); if (old > 0xFFFFFFF0u) atomicAdd((uint32_t*)sm + D * 2 + e, 1u); }
  }
  __syncthreads();
  if (threadIdx.x == 0) atomicAdd((unsigned long long*)out, sm[0]);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  uint64_t *t, *sink; cudaMalloc(&t, 1ull << 32); cudaMalloc(&sink, 8); cudaMemset(t, 0, 1ull << 32);
  const uint64_t n = 1ull << 28;
  float ms;
  for (uint64_t bytes : {16ull << 20, 32ull << 20, 64ull << 20, 128ull << 20, 512ull << 20, 4096ull << 20}) {
    uint64_t slots = bytes / 32, mask = slots - 1;
    k_rand_load<<<sms * 8, 256>>>(t, mask, n, sink);
    cudaEventRecord(a); k_rand_load<<<sms * 8, 256>>>(t, mask, n, sink); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("rand 8B load   table %6llu MB: %7.1f G/s\n", (unsigned long long)(bytes >> 20), n / ms / 1e6);
    k_rand_red<1><<<sms * 8, 256>>>(t, mask, n);
    cudaEventRecord(a); k_rand_red<1><<<sms * 8, 256>>>(t, mask, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("rand RED x1    table %6llu MB: %7.1f G slots/s (%.1f G RED/s)\n", (unsigned long long)(bytes >> 20), n / ms / 1e6, n / ms / 1e6);
    k_rand_red<3><<<sms * 8, 256>>>(t, mask, n);
    cudaEventRecord(a); k_rand_red<3><<<sms * 8, 256>>>(t, mask, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("rand RED x3    table %6llu MB: %7.1f G slots/s (%.1f G RED/s)\n", (unsigned long long)(bytes >> 20), n / ms / 1e6, 3 * n / ms / 1e6);
  }
  for (uint32_t D : {16u, 1024u, 4096u}) {
    size_t sb = (size_t)D * 8 * 3;
    cudaFuncSetAttribute(k_smem<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
    cudaFuncSetAttribute(k_smem<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
    cudaFuncSetAttribute(k_smem<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
    cudaFuncSetAttribute(k_smem<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
    const char* names[4] = {"ATOMS.ADD.32", "u64 add (CAS loop)", "f64 add (CAS loop)", "u32 add + carry"};
    for (int m = 0; m < 4; ++m) {
      auto launch = [&]() {
        if (m == 0) k_smem<0><<<sms * 2, 512, sb>>>(n, D, sink);
        if (m == 1) k_smem<1><<<sms * 2, 512, sb>>>(n, D, sink);
        if (m == 2) k_smem<2><<<sms * 2, 512, sb>>>(n, D, sink);
        if (m == 3) k_smem<3><<<sms * 2, 512, sb>>>(n, D, sink);
      };
      launch();
      cudaEventRecord(a); launch(); cudaEventRecord(b); cudaEventSynchronize(b);
      cudaEventElapsedTime(&ms, a, b);
      printf("smem %-20s D=%5u: %7.1f G ops/s  (%.2f cyc/op/SM @1.95GHz)\n", names[m], D, n / ms / 1e6,
             sms * 1.95e9 / (n / ms * 1e3));
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
