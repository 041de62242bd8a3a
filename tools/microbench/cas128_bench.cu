// cas128_bench.cu — L2 atomic throughput for updating two 8-byte fields of a random 16-byte entry:
//   mode 0: 2 x REDG (u64 add + f64 add)             (what path (b) pass 2 does per field pair)
//   mode 1: 16-byte load + 1 x 128-bit CAS (retry on failure)   (one request for both fields)
//   mode 2: 16-byte load + 2 x REDG
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/cas128 tools/microbench/cas128_bench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t h) {
  h ^= h >> 33; h *= 0xff51afd7ed558ccdull; h ^= h >> 33; h *= 0xc4ceb9fe1a85ec53ull; h ^= h >> 33; return h;
}
__device__ __forceinline__ void cas128(unsigned long long* a, unsigned long long cl, unsigned long long ch,
                                       unsigned long long nl, unsigned long long nh, unsigned long long& ol,
                                       unsigned long long& oh) {
  asm volatile("{\n\t.reg .b128 d, c, n;\n\tmov.b128 c, {%2, %3};\n\tmov.b128 n, {%4, %5};\n\t"
               "atom.global.cas.b128 d, [%6], c, n;\n\tmov.b128 {%0, %1}, d;\n\t}"
               : "=l"(ol), "=l"(oh) : "l"(cl), "l"(ch), "l"(nl), "l"(nh), "l"(a) : "memory");
}
template <int MODE>
__global__ void k(unsigned long long* t, uint64_t mask, uint64_t n, uint64_t seed) {
  uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, st = (uint64_t)gridDim.x * blockDim.x;
  for (; i < n; i += st) {
    uint64_t e = mix(i ^ seed) & mask;
    unsigned long long* p = t + 2 * e;
    if (MODE == 0) {
      atomicAdd(p, 1ull);
      atomicAdd((double*)p + 1, 0.5);
    } else if (MODE == 1) {
      ulonglong2 c = __ldcg((const ulonglong2*)p);
      for (;;) {
        unsigned long long ol, oh;
        double s = __longlong_as_double(c.y) + 0.5;
        cas128(p, c.x, c.y, c.x + 1, __double_as_longlong(s), ol, oh);
        if (ol == c.x && oh == c.y) break;
        c.x = ol; c.y = oh;
      }
    } else {
      ulonglong2 c = __ldcg((const ulonglong2*)p);
      if (c.x != ~0ull) { atomicAdd(p, 1ull); atomicAdd((double*)p + 1, 0.5); }
    }
  }
}
int main() {
  const uint64_t n = 1ull << 28;
  for (uint64_t mb : {16ull, 32ull, 48ull, 512ull}) {
    uint64_t entries = mb * (1ull << 20) / 16;
    unsigned long long* t;
    cudaMalloc(&t, entries * 16);
    cudaMemset(t, 0, entries * 16);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    for (int mode = 0; mode < 3; ++mode) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(a);
        if (mode == 0) k<0><<<148 * 8, 256>>>(t, entries - 1, n, rep);
        if (mode == 1) k<1><<<148 * 8, 256>>>(t, entries - 1, n, rep);
        if (mode == 2) k<2><<<148 * 8, 256>>>(t, entries - 1, n, rep);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (rep) printf("table %4llu MB mode %d (%s): %.1f G updates/s\n", (unsigned long long)mb, mode,
                        mode == 0 ? "2 RED" : mode == 1 ? "ld16 + CAS128" : "ld16 + 2 RED", n / ms / 1e6);
      }
    }
    cudaFree(t);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
