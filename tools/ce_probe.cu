// Copy-engine arbitration probe: stream A queues N x 64 MiB H2D copies; stream B then queues one
// 32 MiB H2D.  When does B's copy finish relative to A's?  For pinned (cudaHostAlloc) and
// registered (mmap + cudaHostRegister) sources, and with stream priorities.
// Build: nvcc -O2 -o build/ce_probe tools/ce_probe.cu
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <cstdio>
#include <cstring>

int main() {
  const size_t C = 64ull << 20, N = 40;
  char *hp, *hr, *d, *d2;
  cudaHostAlloc(&hp, C * N, 0);
  hr = (char*)mmap(nullptr, C * N, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  memset(hr, 1, C * N);
  cudaHostRegister(hr, C * N, cudaHostRegisterPortable);
  cudaMalloc(&d, C * N);
  cudaMalloc(&d2, 32 << 20);
  int lo, hi;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  for (int src = 0; src < 2; ++src)
    for (int prio = 0; prio < 2; ++prio) {
      cudaStream_t a, b;
      cudaStreamCreateWithPriority(&a, cudaStreamNonBlocking, lo);
      cudaStreamCreateWithPriority(&b, cudaStreamNonBlocking, prio ? hi : lo);
      cudaEvent_t e0, ea, eb;
      cudaEventCreate(&e0);
      cudaEventCreate(&ea);
      cudaEventCreate(&eb);
      char* h = src ? hr : hp;
      cudaDeviceSynchronize();
      cudaEventRecord(e0, a);
      for (size_t i = 0; i < N; ++i) cudaMemcpyAsync(d + i * C, h + i * C, C, cudaMemcpyHostToDevice, a);
      cudaEventRecord(ea, a);
      cudaStreamWaitEvent(b, e0, 0);
      cudaMemcpyAsync(d2, h, 32 << 20, cudaMemcpyHostToDevice, b);
      cudaEventRecord(eb, b);
      cudaDeviceSynchronize();
      float ta, tb;
      cudaEventElapsedTime(&ta, e0, ea);
      cudaEventElapsedTime(&tb, e0, eb);
      printf("%s src, B prio %s: A (%zu x 64 MiB) done at %.1f ms, B (32 MiB) done at %.1f ms\n",
             src ? "registered" : "cudaHostAlloc", prio ? "high" : "low ", N, ta, tb);
    }
  return 0;
}
