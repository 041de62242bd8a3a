// Aggregation rate of C3-shaped rows (COUNT + SUM(i64) + SUM(f64)) into shared-memory tables spread
// over a thread-block cluster (DSMEM): each row's key picks an owner CTA of the cluster and an entry
// there; the three updates are atomics on the owner's shared memory (remote for 15/16 of the rows at
// cluster size 16). Rows are synthesised in registers (no memory traffic). Cluster size 1 = the
// local-only rate of the existing bucket tables. Dev tool:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dsmem_agg_bench dsmem_agg_bench.cu
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
namespace cg = cooperative_groups;

constexpr int kEntries = 2048;  // per CTA: count u32 + sum lo/hi u32 + f64 = 20 B -> 40 KB (static limit)

__device__ __forceinline__ uint64_t mix(uint64_t h) {
  h ^= h >> 33; h *= 0xff51afd7ed558ccdull; h ^= h >> 33; h *= 0xc4ceb9fe1a85ec53ull; h ^= h >> 33;
  return h;
}

template <int CS>
__global__ void __launch_bounds__(1024, 1) k_agg(uint64_t rows_per_thread, uint64_t* sink) {
  __shared__ uint32_t cnt[kEntries];
  __shared__ uint32_t slo[kEntries];
  __shared__ uint32_t shi[kEntries];
  __shared__ double sf[kEntries];
  for (int e = threadIdx.x; e < kEntries; e += blockDim.x) { cnt[e] = 0; slo[e] = 0; shi[e] = 0; sf[e] = 0; }
  cg::cluster_group cl = cg::this_cluster();
  if (CS > 1) cl.sync(); else __syncthreads();
  uint64_t s = ((uint64_t)blockIdx.x << 32) ^ threadIdx.x;
  for (uint64_t i = 0; i < rows_per_thread; ++i) {
    const uint64_t h = mix(s + i * 0x9E3779B97F4A7C15ull);
    const uint32_t owner = CS > 1 ? (uint32_t)(h >> 60) % CS : 0;
    const uint32_t e = (uint32_t)(h >> 20) & (kEntries - 1);
    uint32_t* c = CS > 1 ? cl.map_shared_rank(cnt, owner) : cnt;
    uint32_t* lo = CS > 1 ? cl.map_shared_rank(slo, owner) : slo;
    double* f = CS > 1 ? cl.map_shared_rank(sf, owner) : sf;
    atomicAdd(c + e, 1u);
    const uint32_t v = (uint32_t)h;
    const uint32_t old = atomicAdd(lo + e, v);
    if (old + v < old) {
      uint32_t* hi = CS > 1 ? cl.map_shared_rank(shi, owner) : shi;
      atomicAdd(hi + e, 1u);
    }
    atomicAdd(f + e, (double)(h & 1023) / 64.0);
  }
  if (CS > 1) cl.sync(); else __syncthreads();
  uint64_t acc = 0;
  for (int e = threadIdx.x; e < kEntries; e += blockDim.x) acc += cnt[e] + slo[e] + (uint64_t)sf[e];
  atomicAdd((unsigned long long*)sink, (unsigned long long)acc);
}

template <int CS>
void run(uint64_t rpt) {
  uint64_t* sink;
  cudaMalloc(&sink, 8);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto k = k_agg<CS>;
  if (CS > 8) cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  cudaLaunchConfig_t cfg{};
  int grid = (sms / CS) * CS;
  if (CS > 1) {
    int ncl = 0;
    cudaLaunchAttribute a0{};
    a0.id = cudaLaunchAttributeClusterDimension;
    a0.val.clusterDim.x = CS; a0.val.clusterDim.y = 1; a0.val.clusterDim.z = 1;
    cudaLaunchConfig_t q{};
    q.gridDim = dim3(CS); q.blockDim = dim3(1024); q.attrs = &a0; q.numAttrs = 1;
    cudaOccupancyMaxActiveClusters(&ncl, k, &q);
    grid = ncl * CS;
  }
  cudaLaunchAttribute attr{};
  attr.id = cudaLaunchAttributeClusterDimension;
  attr.val.clusterDim.x = CS; attr.val.clusterDim.y = 1; attr.val.clusterDim.z = 1;
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(1024);
  cfg.attrs = &attr;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, k, rpt, sink);
  cudaDeviceSynchronize();
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  cudaLaunchKernelEx(&cfg, k, rpt, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  const double rows = (double)grid * 1024 * rpt;
  printf("cluster %2d: grid %d CTAs, %.1f G rows/s (%s)\n", CS, grid, rows / ms / 1e6,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  const uint64_t rpt = 4096;
  run<1>(rpt);
  run<2>(rpt);
  run<4>(rpt);
  run<8>(rpt);
  run<16>(rpt);
  return 0;
}
