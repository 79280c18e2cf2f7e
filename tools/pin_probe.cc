// Probe: how fast can N GiB of host memory be page-locked on this box?
//   (a) cudaHostAlloc(Portable|Mapped)
//   (b) mmap + T threads first-touching their ranges + cudaHostRegister(Portable|Mapped)
//   (c) like (b) but with MAP_POPULATE instead of threads
// and H2D/D2H copy bandwidth from the (b) buffer.  Build: nvcc -O2 -o build/pin_probe tools/pin_probe.cc
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

#define CK(x)                                                              \
  do {                                                                     \
    cudaError_t e = (x);                                                   \
    if (e != cudaSuccess) {                                                \
      printf("%s: %s\n", #x, cudaGetErrorString(e));                       \
      exit(1);                                                             \
    }                                                                      \
  } while (0)

int main(int argc, char** argv) {
  const size_t gib = argc > 1 ? atoi(argv[1]) : 16;
  const int T = argc > 2 ? atoi(argv[2]) : 16;
  const size_t n = gib << 30;
  CK(cudaFree(0));
  double t0 = now();
  void* a;
  CK(cudaHostAlloc(&a, n, cudaHostAllocPortable | cudaHostAllocMapped));
  double t1 = now();
  printf("(a) cudaHostAlloc %zu GiB: %.2f s (%.1f GB/s)\n", gib, t1 - t0, n / (t1 - t0) / 1e9);
  CK(cudaFreeHost(a));

  t0 = now();
  char* b = (char*)mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  madvise(b, n, MADV_HUGEPAGE);
  std::vector<std::thread> th;
  for (int i = 0; i < T; ++i)
    th.emplace_back([=] {
      for (size_t o = n * i / T; o < n * (i + 1) / T; o += 4096) b[o] = 0;
    });
  for (auto& x : th) x.join();
  double t2 = now();
  CK(cudaHostRegister(b, n, cudaHostRegisterPortable | cudaHostRegisterMapped));
  double t3 = now();
  printf("(b) mmap+%d-thread touch %.2f s + cudaHostRegister %.2f s = %.2f s (%.1f GB/s)\n", T, t2 - t0, t3 - t2,
         t3 - t0, n / (t3 - t0) / 1e9);
  void* d;
  CK(cudaMalloc(&d, 1ull << 30));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int dir = 0; dir < 2; ++dir) {
    cudaEventRecord(e0);
    for (int k = 0; k < 4; ++k)
      CK(cudaMemcpyAsync(dir ? (void*)(b + (size_t(k) << 30)) : d, dir ? d : (void*)(b + (size_t(k) << 30)), 1ull << 30,
                         dir ? cudaMemcpyDeviceToHost : cudaMemcpyHostToDevice));
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("    %s from registered buffer: %.1f GB/s\n", dir ? "D2H" : "H2D", 4.0 * (1 << 30) / (ms * 1e6));
  }
  CK(cudaHostUnregister(b));
  munmap(b, n);

  t0 = now();
  char* c = (char*)mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS | MAP_POPULATE, -1, 0);
  double t4 = now();
  CK(cudaHostRegister(c, n, cudaHostRegisterPortable | cudaHostRegisterMapped));
  double t5 = now();
  printf("(c) mmap(MAP_POPULATE) %.2f s + cudaHostRegister %.2f s = %.2f s\n", t4 - t0, t5 - t4, t5 - t0);
  CK(cudaHostUnregister(c));
  munmap(c, n);
  return 0;
}
