// Probe: H2D/D2H overlap with a static cudart, host memory from cudaHostAlloc
// (own) vs cudaHostRegister'ed malloc -- diagnoses abft_spmv_host_pipelined.
#include <cstdio>
#include <cstdlib>
#include <chrono>
#include <cuda_runtime.h>
__global__ void touch(double *y, const double *x, size_t n) {
  for (size_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) y[i] = x[i] * 2.0;
}
int main() {
  const size_t n = 2u << 20, B = n * 8;
  double *xh, *yh, *px[2], *py[2];
  cudaHostAlloc(&xh, B, 0); cudaHostAlloc(&yh, B, 0);
  for (int q = 0; q < 2; ++q) { cudaMalloc(&px[q], B); cudaMalloc(&py[q], B); }
  cudaStream_t s, si, so; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&si, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&so, cudaStreamNonBlocking);
  cudaEvent_t ex[2], ec[2], eo[2];
  for (int q = 0; q < 2; ++q) { cudaEventCreateWithFlags(&ex[q], cudaEventDisableTiming); cudaEventCreateWithFlags(&ec[q], cudaEventDisableTiming); cudaEventCreateWithFlags(&eo[q], cudaEventDisableTiming); }
  for (int rep = 0; rep < 2; ++rep) {
    const int K = 100;
    cudaDeviceSynchronize();
    auto t0 = std::chrono::steady_clock::now();
    for (int k = 0; k < K; ++k) {
      int sl = k & 1;
      if (k >= 2) cudaStreamWaitEvent(si, ec[sl], 0);
      cudaMemcpyAsync(px[sl], xh, B, cudaMemcpyHostToDevice, si);
      cudaEventRecord(ex[sl], si);
      cudaStreamWaitEvent(s, ex[sl], 0);
      if (k >= 2) cudaStreamWaitEvent(s, eo[sl], 0);
      touch<<<1184, 256, 0, s>>>(py[sl], px[sl], n);
      cudaEventRecord(ec[sl], s);
      cudaStreamWaitEvent(so, ec[sl], 0);
      cudaMemcpyAsync(yh, py[sl], B, cudaMemcpyDeviceToHost, so);
      cudaEventRecord(eo[sl], so);
    }
    cudaDeviceSynchronize();
    double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count() / K;
    printf("pipelined %.4f ms/step (%s)\n", ms, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
