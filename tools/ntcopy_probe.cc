// Staged-weight fill: glibc memcpy vs non-temporal (streaming) stores, pageable -> pinned, T threads,
// 8 MiB copies (the fill-part granularity), alone and while a copy engine streams H2D from the
// pinned buffer.  A regular store reads the destination line first (read-for-ownership), so the
// staged path costs 4 DRAM passes per byte (src read, dst RFO, dst write, DMA read); streaming
// stores skip the RFO (3 passes).  glibc only switches to streaming stores above
// __x86_shared_non_temporal_threshold, typically larger than one 8 MiB part.
// Build: nvcc -O2 -o build/ntcopy_probe tools/ntcopy_probe.cc -lpthread
#include <cuda_runtime.h>
#include <emmintrin.h>
#include <sys/mman.h>

#include <atomic>
#include <chrono>
#include <cstdint>
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

static void nt_copy(char* dst, const char* src, size_t n) {
  size_t i = 0;
  while (i < n && ((uintptr_t(dst) + i) & 63)) dst[i] = src[i], ++i;
  for (; i + 64 <= n; i += 64) {
    __m128i a = _mm_loadu_si128((const __m128i*)(src + i));
    __m128i b = _mm_loadu_si128((const __m128i*)(src + i + 16));
    __m128i c = _mm_loadu_si128((const __m128i*)(src + i + 32));
    __m128i d = _mm_loadu_si128((const __m128i*)(src + i + 48));
    _mm_stream_si128((__m128i*)(dst + i), a);
    _mm_stream_si128((__m128i*)(dst + i + 16), b);
    _mm_stream_si128((__m128i*)(dst + i + 32), c);
    _mm_stream_si128((__m128i*)(dst + i + 48), d);
  }
  for (; i < n; ++i) dst[i] = src[i];
  _mm_sfence();
}

int main() {
  const size_t C = 8ull << 20, SRC = 8ull << 30, DST = 2ull << 30;
  char* src = anon(SRC, false);
  char* dst = anon(DST, true);
  cudaHostRegister(dst, DST, cudaHostRegisterPortable | cudaHostRegisterMapped);
  char* dev;
  cudaMalloc(&dev, DST);
  for (int rep = 0; rep < 2; ++rep)
    for (int with_dma = 0; with_dma < 2; ++with_dma)
      for (int nt = 0; nt < 2; ++nt)
        for (int T : {8, 12, 16}) {
          std::atomic<bool> stop{false};
          std::atomic<uint64_t> dma_bytes{0};
          std::thread dma;
          if (with_dma)
            dma = std::thread([&] {
              cudaStream_t s;
              cudaStreamCreate(&s);
              while (!stop) {
                cudaMemcpyAsync(dev, dst, 256ull << 20, cudaMemcpyHostToDevice, s);
                cudaStreamSynchronize(s);
                dma_bytes += 256ull << 20;
              }
            });
          const int per = 48;
          double t0 = now();
          std::vector<std::thread> th;
          for (int t = 0; t < T; ++t)
            th.emplace_back([&, t] {
              for (int i = 0; i < per; ++i) {
                const size_t k = size_t(t) * per + i;
                char* d = dst + (k * C) % (DST - C);
                const char* s = src + (k * C) % (SRC - C);
                if (nt)
                  nt_copy(d, s, C);
                else
                  memcpy(d, s, C);
              }
            });
          for (auto& x : th) x.join();
          double dt = now() - t0;
          stop = true;
          if (with_dma) dma.join();
          printf("rep %d %s %s T=%2d: fill %5.1f GB/s  concurrent H2D %5.1f GB/s\n", rep, nt ? "stream" : "memcpy",
                 with_dma ? "+H2D" : "    ", T, double(T) * per * C / dt / 1e9, dma_bytes / dt / 1e9);
          fflush(stdout);
        }
  return 0;
}
