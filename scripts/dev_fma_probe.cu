// Dev: FP64 FMA-throughput probe variants (is stencil_fma_probe's 34.2 TFLOP/s
// the hardware's sustained rate?). nvcc -gencode arch=compute_100a,code=sm_100a
// -O3 -o /tmp/fmaprobe scripts/dev_fma_probe.cu && /tmp/fmaprobe
#include <cstdio>
#include <cuda_runtime.h>

template <int NACC, bool IMM>
__global__ void __launch_bounds__(256) probe(double* sink, long long iters, double a, double b) {
  double x[NACC];
#pragma unroll
  for (int k = 0; k < NACC; ++k) x[k] = (threadIdx.x + k) * 1e-3;
  for (long long i = 0; i < iters; ++i) {
#pragma unroll
    for (int u = 0; u < 8; ++u)
#pragma unroll
      for (int k = 0; k < NACC; ++k) x[k] = IMM ? fma(x[k], 0.9990234375, 0.0009765625) : fma(x[k], a, b);
  }
  double s = 0;
#pragma unroll
  for (int k = 0; k < NACC; ++k) s += x[k];
  if (s == -12345.0) sink[0] = s;
}

template <int NACC, bool IMM>
void run(double* sink, int bps) {
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const long long iters = 20000;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 20; ++r) {
    cudaEventRecord(e0);
    probe<NACC, IMM><<<nsm * bps, 256>>>(sink, iters, 0.9990234375, 0.0009765625);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 2 && ms < best) best = ms;
  }
  const double fl = 2.0 * nsm * bps * 256.0 * iters * 8 * NACC;
  printf("NACC=%2d IMM=%d blocks/SM=%d: %.2f TFLOP/s (best of 18, %.2f ms)\n", NACC, IMM, bps, fl / (best * 1e-3) / 1e12,
         best);
}

int main() {
  double* sink;
  cudaMalloc(&sink, 8);
  run<8, false>(sink, 8); run<8, true>(sink, 8); run<4, false>(sink, 8); run<16, false>(sink, 8);
  run<16, true>(sink, 8); run<8, false>(sink, 4); run<12, true>(sink, 8); run<8, false>(sink, 8);
  return 0;
}
