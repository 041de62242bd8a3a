// gen.cu — libblugen.so: the seeded synthetic-column generator (bench/test input only).
// It evaluates include/blu_gen.h per element on the host or on the device; it contains no
// GROUP BY arithmetic and is not part of libblugby.
#include <cuda_runtime.h>
#include "blu_gen.h"

namespace {

template <typename T>
__global__ void __launch_bounds__(256) gen_kernel(blu_gen_spec_t s, uint64_t row0, uint64_t n, T* out) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        uint64_t b = blu_gen_bits(&s, row0 + i);
        if constexpr (sizeof(T) == 4) out[i] = (T)(uint32_t)b;
        else out[i] = (T)b;
    }
}

}  // namespace

extern "C" int blu_gen_fill_host(const blu_gen_spec_t* spec, uint64_t row0, uint64_t n, void* out) {
    if (!spec || (!out && n)) return 1;
    blu_gen_fill_host_inline(spec, row0, n, out);
    return 0;
}

extern "C" int blu_gen_fill_device(const blu_gen_spec_t* spec, uint64_t row0, uint64_t n, void* out,
                                   void* stream) {
    if (!spec || (!out && n)) return 1;
    if (n == 0) return 0;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint64_t blocks = (n + 255) / 256;
    uint64_t cap = (uint64_t)sms * 16;
    if (blocks > cap) blocks = cap;
    cudaStream_t st = (cudaStream_t)stream;
    if (spec->dtype == BLU_GEN_I32)
        gen_kernel<int32_t><<<(unsigned)blocks, 256, 0, st>>>(*spec, row0, n, (int32_t*)out);
    else
        gen_kernel<uint64_t><<<(unsigned)blocks, 256, 0, st>>>(*spec, row0, n, (uint64_t*)out);
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

extern "C" void blu_gen_zipf_table(uint64_t n, double s, uint64_t* out) { blu_gen_zipf_table_host(n, s, out); }

extern "C" void blu_gen_permutation(uint64_t n, uint64_t seed, uint32_t* out) {
    blu_gen_permutation_host(n, seed, out);
}
