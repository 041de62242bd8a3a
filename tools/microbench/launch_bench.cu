// Host cost of one kernel launch vs the kernel-parameter size and the launch path (dev tool):
// <<<>>> of a static kernel with a 3.3 KB / 256 B / 16 B parameter block, and the same 3.3 KB kernel
// loaded from a cubin with cudaLibraryLoadData and launched through its cudaKernel_t (the NVRTC path
// of libblugby). nvcc -gencode arch=compute_100a,code=sm_100a -o launch_bench launch_bench.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <vector>
template <int B>
struct P { unsigned char b[B]; };
template <int B>
__global__ void k(P<B> p, int* out) { if (threadIdx.x == 0 && p.b[0] == 7) out[0] = p.b[B - 1]; }

template <class F>
double per_launch_us(F f, int n) {
  for (int i = 0; i < 100; ++i) f();
  cudaDeviceSynchronize();
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) f();
  auto t1 = std::chrono::steady_clock::now();
  cudaDeviceSynchronize();
  return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}
int main() {
  int* out;
  cudaMalloc(&out, 64);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  P<3328> big{};
  P<256> mid{};
  P<16> small{};
  const int n = 2000;
  printf("<<<>>> 3328 B params: %.2f us\n", per_launch_us([&] { k<3328><<<296, 512, 0, st>>>(big, out); }, n));
  printf("<<<>>>  256 B params: %.2f us\n", per_launch_us([&] { k<256><<<296, 512, 0, st>>>(mid, out); }, n));
  printf("<<<>>>   16 B params: %.2f us\n", per_launch_us([&] { k<16><<<296, 512, 0, st>>>(small, out); }, n));
  void* args[] = {&big, &out};
  printf("cudaLaunchKernel 3328 B: %.2f us\n", per_launch_us([&] {
    cudaLaunchKernel((const void*)k<3328>, dim3(296), dim3(512), args, 0, st); }, n));
  // launch + 16-byte D2H + sync: the small-query critical path without any kernel work
  int h[4];
  printf("launch(3328 B) + D2H 16 B + sync: %.2f us\n", per_launch_us([&] {
    k<3328><<<296, 512, 0, st>>>(big, out);
    cudaMemcpyAsync(h, out, 16, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st); }, 500));
  printf("launch(16 B) + D2H 16 B + sync: %.2f us\n", per_launch_us([&] {
    k<16><<<296, 512, 0, st>>>(small, out);
    cudaMemcpyAsync(h, out, 16, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st); }, 500));
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  k<3328><<<296, 512, 0, st>>>(big, out);
  cudaMemcpyAsync(h, out, 16, cudaMemcpyDeviceToHost, st);
  cudaStreamEndCapture(st, &g);
  cudaGraphInstantiate(&ge, g, 0);
  printf("graph(launch 3328 B + D2H) + sync: %.2f us\n", per_launch_us([&] {
    cudaGraphLaunch(ge, st);
    cudaStreamSynchronize(st); }, 500));
  // the NVRTC path: a cubin loaded as a cudaLibrary, launched through its cudaKernel_t, and the
  // same kernel's CUfunction (cuKernelGetFunction) through the driver's cuLaunchKernel
  if (FILE* f = fopen("tools/microbench/lk_cubin.bin", "rb")) {
    std::vector<char> cub;
    fseek(f, 0, SEEK_END);
    cub.resize(ftell(f));
    fseek(f, 0, SEEK_SET);
    if (fread(cub.data(), 1, cub.size(), f) != cub.size()) return 1;
    fclose(f);
    cudaLibrary_t lib;
    cudaKernel_t kk;
    cudaLibraryLoadData(&lib, cub.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
    cudaLibraryGetKernel(&kk, lib, "k3328");
    printf("cudaKernel_t cudaLaunchKernel 3328 B: %.2f us\n", per_launch_us([&] {
      cudaLaunchKernel((const void*)kk, dim3(296), dim3(512), args, 0, st); }, n));
    CUfunction fn;
    if (cuKernelGetFunction(&fn, (CUkernel)kk) == CUDA_SUCCESS) {
      printf("CUfunction cuLaunchKernel 3328 B: %.2f us\n", per_launch_us([&] {
        cuLaunchKernel(fn, 296, 1, 1, 512, 1, 1, 0, (CUstream)st, args, nullptr); }, n));
    }
  }
  return 0;
}
