// Host-side ceiling of the staged weight path: pageable -> pinned memcpy bandwidth with T threads
// (8 MiB copies, the fill-part granularity), alone and while a copy engine streams H2D from the
// pinned buffer, for pinned buffers made by cudaHostAlloc vs mmap(+THP)+cudaHostRegister, and for
// sources with and without transparent huge pages.
// Build: nvcc -O2 -o build/memcpy_probe tools/memcpy_probe.cc -lpthread
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <thread>
#include <vector>

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

static char* anon(size_t n, bool thp) {
  char* p = (char*)mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  madvise(p, n, thp ? MADV_HUGEPAGE : MADV_NOHUGEPAGE);
  memset(p, 1, n);
  return p;
}

int main() {
  const size_t C = 8ull << 20, SRC = 8ull << 30, DST = 2ull << 30;
  char* src_thp = anon(SRC, true);
  char* src_4k = anon(SRC, false);
  char* dst_alloc;
  cudaHostAlloc(&dst_alloc, DST, 0);
  memset(dst_alloc, 0, DST);
  char* dst_reg = anon(DST, true);
  cudaHostRegister(dst_reg, DST, cudaHostRegisterPortable | cudaHostRegisterMapped);
  char* dev;
  cudaMalloc(&dev, DST);
  struct V {
    const char* name;
    char* src;
    char* dst;
  };
  for (V v : {V{"src THP, dst cudaHostAlloc ", src_thp, dst_alloc}, V{"src THP, dst mmap+register", src_thp, dst_reg},
              V{"src 4K,  dst cudaHostAlloc ", src_4k, dst_alloc}, V{"src 4K,  dst mmap+register", src_4k, dst_reg}})
    for (int with_dma = 0; with_dma < 2; ++with_dma)
      for (int T : {8, 12, 16}) {
        std::atomic<bool> stop{false};
        std::thread dma;
        if (with_dma)
          dma = std::thread([&] {
            cudaStream_t s;
            cudaStreamCreate(&s);
            while (!stop) {
              cudaMemcpyAsync(dev, v.dst, DST, cudaMemcpyHostToDevice, s);
              cudaStreamSynchronize(s);
            }
          });
        const int per = 64;
        double t0 = now();
        std::vector<std::thread> th;
        for (int t = 0; t < T; ++t)
          th.emplace_back([&, t] {
            for (int i = 0; i < per; ++i) {
              const size_t k = size_t(t) * per + i;
              memcpy(v.dst + (k * C) % (DST - C), v.src + (k * C) % (SRC - C), C);
            }
          });
        for (auto& x : th) x.join();
        double dt = now() - t0;
        stop = true;
        if (with_dma) dma.join();
        printf("%s %s T=%2d: %5.1f GB/s\n", v.name, with_dma ? "+H2D" : "    ", T, double(T) * per * C / dt / 1e9);
        fflush(stdout);
      }
  return 0;
}
