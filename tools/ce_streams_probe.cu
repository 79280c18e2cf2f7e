// Does splitting each PCIe direction over several copy-engine streams raise the duplex ceiling?
// 1 GiB per direction (pinned host <-> device), as 1 / 2 / 4 equal slices on that many streams per
// direction, alone and with both directions at once.  GB/s over the union of the intervals.
// Build: nvcc -O3 -o /tmp/cesp tools/ce_streams_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

int main() {
  const size_t n = 1ull << 30;
  char *h1, *h2, *d1, *d2;
  cudaHostAlloc(&h1, n, cudaHostAllocPortable);
  cudaHostAlloc(&h2, n, cudaHostAllocPortable);
  cudaMalloc(&d1, n);
  cudaMalloc(&d2, n);
  std::vector<cudaStream_t> s(8);
  for (auto& x : s) cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int dirs : {1, 2, 3}) {  // 1 = D2H only, 2 = H2D only, 3 = both
    for (int k : {1, 2, 4}) {
      float best = 1e9f;
      for (int r = 0; r < 5; ++r) {
        cudaDeviceSynchronize();
        cudaEventRecord(a, s[0]);
        for (int i = 1; i < 8; ++i) cudaStreamWaitEvent(s[i], a, 0);
        const size_t sl = n / k;
        for (int i = 0; i < k; ++i) {
          if (dirs & 1) cudaMemcpyAsync(h1 + i * sl, d1 + i * sl, sl, cudaMemcpyDeviceToHost, s[i]);
          if (dirs & 2) cudaMemcpyAsync(d2 + i * sl, h2 + i * sl, sl, cudaMemcpyHostToDevice, s[4 + i]);
        }
        for (int i = 1; i < 8; ++i) {
          cudaEvent_t e;
          cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
          cudaEventRecord(e, s[i]);
          cudaStreamWaitEvent(s[0], e, 0);
          cudaEventDestroy(e);
        }
        cudaEventRecord(b, s[0]);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r) best = std::min(best, ms);
      }
      const double bytes = (dirs == 3 ? 2.0 : 1.0) * n;
      printf("%-8s streams/direction %d: %.1f GB/s\n", dirs == 1 ? "D2H" : dirs == 2 ? "H2D" : "duplex", k,
             bytes / (best * 1e6));
    }
  }
  return 0;
}
