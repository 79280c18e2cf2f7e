// Host-side ceiling of the staged weight path: pageable -> pinned memcpy bandwidth with T threads
// (64 MiB chunks, the Stage Buffer granularity), alone and while a copy engine streams H2D from
// the pinned buffer.  Build: nvcc -O2 -o build/memcpy_probe tools/memcpy_probe.cc -lpthread
#include <cuda_runtime.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <thread>
#include <vector>

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  const size_t C = 64ull << 20, SRC = 8ull << 30, DST = 2ull << 30;
  char* src = new char[SRC];
  memset(src, 1, SRC);
  char* dst;
  cudaHostAlloc(&dst, DST, 0);
  memset(dst, 0, DST);
  char* dev;
  cudaMalloc(&dev, DST);
  for (int with_dma = 0; with_dma < 2; ++with_dma) {
    for (int T : {1, 4, 8, 12, 16}) {
      std::atomic<bool> stop{false};
      std::thread dma;
      if (with_dma)
        dma = std::thread([&] {
          cudaStream_t s;
          cudaStreamCreate(&s);
          while (!stop) {
            cudaMemcpyAsync(dev, dst, DST, cudaMemcpyHostToDevice, s);
            cudaStreamSynchronize(s);
          }
        });
      const int per = 24;  // chunks per thread
      double t0 = now();
      std::vector<std::thread> th;
      for (int t = 0; t < T; ++t)
        th.emplace_back([&, t] {
          for (int i = 0; i < per; ++i) {
            const size_t so = (size_t(t) * per + i) * C % (SRC - C), d = (size_t(t) * per + i) * C % (DST - C);
            memcpy(dst + d, src + so, C);
          }
        });
      for (auto& x : th) x.join();
      double dt = now() - t0;
      stop = true;
      if (with_dma) dma.join();
      printf("%s T=%2d: %.1f GB/s pageable->pinned\n", with_dma ? "with H2D DMA" : "alone       ", T,
             double(T) * per * C / dt / 1e9);
    }
  }
  return 0;
}
