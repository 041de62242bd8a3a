// kmv.cu — on-GPU KMV ("K-minimum values") estimate of the number of groups.
//
// The paper computes the estimate on CPU threads right after the HASH evaluator: "We use CPU threads
// to load data and then use a simple hash function and KMV[2] algorithm to estimate the number of
// groups. We will use this estimate to tune the size of the GPU data structures." (also P:127).
// Here it runs on the device over the key columns already in HBM:
//   h(row) = fmix64(packed_key ^ kKmvSalt)            (independent of the table's slot hash)
//   L      = the k smallest DISTINCT values of h over all rows
//   est    = (k - 1) * 2^64 / L[k-1]                   (exact distinct count if fewer than k)
// (the same definition is written out plainly in oracle/kmv_oracle.cpp, which the tests compare with)
// Each CTA keeps its k smallest distinct hashes in shared memory (a row survives only if it is below
// the CTA's current k-th value; survivors are buffered and merged with a bitonic sort); the per-CTA
// lists are then merged by one device sort (the repo's own LSD radix sort, sort.cu). The result depends only on the SET of keys, not on the
// row order or the launch shape.
#include <cuda_runtime.h>
#include <stdint.h>

#include "blu_internal.h"
#include "blu_device.cuh"

namespace blu {

constexpr uint64_t kKmvSalt = 0x6b6d765f73616c74ull;  // "kmv_salt"
constexpr uint32_t kKmvMaxK = 2048;
constexpr uint32_t kKmvBuf = 4096;   // survivor buffer (a tile adds at most 2048)
constexpr uint32_t kKmvSort = 8192;  // L (k) + buffer (<= kKmvBuf) padded to a power of two

// Bitonic sort of n (power of two) u64 in shared memory, ascending.
__device__ void bitonic_sort_smem(uint64_t* a, uint32_t n) {
  for (uint32_t size = 2; size <= n; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < n / 2; i += blockDim.x) {
        const uint32_t lo = 2 * stride * (i / stride) + (i % stride), hi = lo + stride;
        const bool up = (lo & size) == 0;
        const uint64_t x = a[lo], y = a[hi];
        if ((x > y) == up) {
          a[lo] = y;
          a[hi] = x;
        }
      }
    }
  }
  __syncthreads();
}

// Merge the survivor buffer into L: sort L ∪ buffer, drop duplicates, keep the k smallest.
__device__ void kmv_merge(uint64_t* work, uint32_t* nl, uint32_t* nb, uint32_t k, uint64_t* thr) {
  // work[0, k) = L (sorted, UINT64_MAX padded), work[k, k + nb) = buffer; pad the rest
  const uint32_t used = k + *nb;
  uint32_t n = 1;
  while (n < used) n <<= 1;
  for (uint32_t i = used + threadIdx.x; i < n; i += blockDim.x) work[i] = UINT64_MAX;
  bitonic_sort_smem(work, n);
  // unique-compact the sorted array into the first positions (single warp keeps it simple & ordered)
  if (threadIdx.x < 32) {
    uint32_t out = 0;
    uint64_t carry = 0;  // last element of the previous 32-chunk (read before any write)
    for (uint32_t base = 0; base < n && out < k; base += 32) {
      const uint32_t i = base + threadIdx.x;
      const uint64_t x = i < n ? work[i] : UINT64_MAX;
      uint64_t prev = __shfl_up_sync(0xffffffffu, x, 1);
      if (threadIdx.x == 0) prev = carry;
      carry = __shfl_sync(0xffffffffu, x, 31);
      const bool keep = x != UINT64_MAX && (i == 0 || x != prev);
      const unsigned bal = __ballot_sync(0xffffffffu, keep);  // all reads of this chunk are done
      const uint32_t pos = out + __popc(bal & ((1u << threadIdx.x) - 1u));
      if (keep && pos < k) work[pos] = x;  // pos <= i < later chunks' indices: in-place compaction is safe
      out += __popc(bal);
      __syncwarp();
    }
    if (out > k) out = k;
    for (uint32_t i = out + threadIdx.x; i < k; i += 32) work[i] = UINT64_MAX;
    if (threadIdx.x == 0) {
      *nl = out;
      *nb = 0;
      *thr = out == k ? work[k - 1] : UINT64_MAX;
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(512) k_kmv_local(AggParams p, uint32_t k, uint64_t* cand) {
  extern __shared__ __align__(16) uint64_t work[];  // kKmvSort
  __shared__ uint32_t nl, nb;
  __shared__ uint64_t thr;
  for (uint32_t i = threadIdx.x; i < kKmvSort; i += blockDim.x) work[i] = UINT64_MAX;
  if (threadIdx.x == 0) {
    nl = 0;
    nb = 0;
    thr = UINT64_MAX;
  }
  __syncthreads();
  constexpr int R = 4;
  const uint64_t pol = evict_first_policy();
  const uint64_t n = p.n_rows;
  const uint64_t tile = (uint64_t)blockDim.x * R;
  const uint64_t ntiles = (n + tile - 1) / tile;
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const uint64_t row = lane_base<R>(t * tile, threadIdx.x >> 5, threadIdx.x & 31);
    uint64_t key[R];
    const uint32_t valid = pack_keys<GenericSpec, R>(p, row, n, pol, key);
    const uint64_t th = thr;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!(valid >> r & 1)) continue;
      const uint64_t h = fmix64(key[r] ^ kKmvSalt);
      if (h < th && h != UINT64_MAX) work[k + atomicAdd(&nb, 1u)] = h;
    }
    __syncthreads();
    const bool do_merge = nb > kKmvBuf - tile;  // keep room for the next tile's survivors
    __syncthreads();                             // every thread has read nb before anyone appends again
    if (do_merge) kmv_merge(work, &nl, &nb, k, &thr);
  }
  __syncthreads();
  if (nb) kmv_merge(work, &nl, &nb, k, &thr);
  for (uint32_t i = threadIdx.x; i < k; i += blockDim.x) cand[(uint64_t)blockIdx.x * k + i] = work[i];
}

// sorted candidates -> number of distinct values (capped at k) and the k-th smallest distinct value
__global__ void k_kmv_select(const uint64_t* sorted, uint64_t m, uint32_t k, uint64_t* out /* [count, kth] */) {
  if (threadIdx.x >= 32) return;
  uint64_t cnt = 0, kth = UINT64_MAX;
  for (uint64_t base = 0; base < m && cnt < k; base += 32) {
    const uint64_t i = base + threadIdx.x;
    const uint64_t x = i < m ? sorted[i] : UINT64_MAX;
    const bool keep = x != UINT64_MAX && (i == 0 || x != sorted[i - 1]);
    const unsigned bal = __ballot_sync(0xffffffffu, keep);
    const uint64_t pos = cnt + __popc(bal & ((1u << threadIdx.x) - 1u));
    if (keep && pos == k - 1) kth = x;
    cnt += __popc(bal);
  }
  // lane holding the k-th distinct value (if any) publishes it
  uint64_t found = kth;
  for (int o = 16; o; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, found, o);
    found = y < found ? y : found;
  }
  if (threadIdx.x == 0) {
    out[0] = cnt < k ? cnt : k;
    out[1] = found;
  }
}

}  // namespace blu

using namespace blu;

extern "C" blu_status_t blu_gby_estimate_groups(const blu_key_desc_t* keys, int32_t n_keys, const void* const* key_cols,
                                                uint64_t n_rows, uint32_t k, void* stream, double* est,
                                                int32_t* exact) {
  env_snapshot();
  if (!keys || n_keys < 1 || n_keys > kMaxKeys || !est) return fail(BLU_E_INVALID, "bad estimate arguments");
  if (k < 16 || k > kKmvMaxK) return fail(BLU_E_INVALID, "k must be in [16, %u]", kKmvMaxK);
  if (n_rows && !key_cols) return fail(BLU_E_INVALID, "NULL key columns");
  bool sparse = false;
  uint64_t D = 1;
  AggParams p{};
  p.lay.n_keys = n_keys;
  for (int j = 0; j < n_keys; ++j) {
    if (keys[j].dtype != BLU_I32 && keys[j].dtype != BLU_I64) return fail(BLU_E_INVALID, "key dtype");
    if (keys[j].dict_size == 0) sparse = true;
    p.lay.key_dtype[j] = keys[j].dtype;
    p.lay.dict[j] = keys[j].dict_size;
    p.lay.stride[j] = D;
    if (keys[j].dict_size) {
      if (D > ((1ull << 62) / keys[j].dict_size)) return fail(BLU_E_UNSUPPORTED, "dense key domain >= 2^62");
      D *= keys[j].dict_size;
    }
  }
  if (sparse && n_keys > 1) return fail(BLU_E_UNSUPPORTED, "a sparse key must be the only key column");
  *est = 0;
  if (exact) *exact = 1;
  if (n_rows == 0) return BLU_OK;
  p.lay.sparse = sparse ? 1 : 0;
  p.lay.domain = sparse ? 0 : D;
  bool vec = true;
  for (int j = 0; j < n_keys; ++j) {
    p.key[j] = key_cols[j];
    vec = vec && ((uintptr_t)key_cols[j] & 15) == 0;
  }
  p.vec_ok = vec;
  p.n_rows = n_rows;
  cudaStream_t st = (cudaStream_t)stream;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint32_t grid = (uint32_t)sms;
  const uint64_t m = (uint64_t)grid * k;
  const size_t tmp_bytes = sort_u64_scratch_bytes(m);
  void* ws = nullptr;
  const size_t bytes = 64 + 2 * m * 8 + tmp_bytes;
  if (cudaMallocAsync(&ws, bytes, st) != cudaSuccess) {
    cudaGetLastError();
    return fail(BLU_E_OOM, "estimate workspace");
  }
  uint32_t* flags = (uint32_t*)ws;
  uint64_t* res = (uint64_t*)((uint8_t*)ws + 16);
  uint64_t* cand = (uint64_t*)((uint8_t*)ws + 64);
  uint64_t* sorted = cand + m;
  void* tmp = sorted + m;
  cudaMemsetAsync(ws, 0, 64, st);
  p.flags = flags;
  const size_t smem = kKmvSort * 8;
  cudaFuncSetAttribute(k_kmv_local, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k_kmv_local<<<grid, 512, smem, st>>>(p, k, cand);
  count_launch(1);
  cudaError_t se = sort_u64_keys(cand, sorted, m, tmp, st);
  if (se != cudaSuccess) {
    cudaGetLastError();
    cudaFreeAsync(ws, st);
    return fail(BLU_E_CUDA, "estimate sort: %s", cudaGetErrorString(se));
  }
  k_kmv_select<<<1, 32, 0, st>>>(sorted, m, k, res);
  count_launch(1);
  uint64_t h[4] = {0, 0, 0, 0};
  cudaMemcpyAsync(h, ws, 32, cudaMemcpyDeviceToHost, st);
  cudaError_t e = cudaStreamSynchronize(st);
  cudaFreeAsync(ws, st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(BLU_E_CUDA, "estimate: %s", cudaGetErrorString(e));
  }
  if ((uint32_t)h[0] & FLAG_KEY_RANGE) return fail(BLU_E_KEY_RANGE, "a key code is outside its dictionary");
  const uint64_t cnt = h[2], kth = h[3];
  if (cnt < k) {  // fewer than k distinct hashes: exact
    *est = (double)cnt;
    if (exact) *exact = 1;
  } else {
    *est = (double)(k - 1) * 18446744073709551616.0 / (double)kth;
    if (exact) *exact = 0;
  }
  return BLU_OK;
}
