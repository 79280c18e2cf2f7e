// Where do the ~36 us per launch go?  Event-bracketed durations of the product copy kernel
// (csrc/kernels/copy.cu, included verbatim) in four settings:
//   A back-to-back launches on one stream
//   B each launch after the GPU idled ~2 ms (host sleep)
//   C each launch after a cudaStreamWaitEvent on an event recorded behind a 32 MiB D2H on another stream
//   D like C, but the timing start event is recorded BEFORE the cross-stream wait resolves
// plus the in-kernel %globaltimer span (first CTA start -> last CTA end) for A/B/C.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -o build/launch_probe tools/launch_probe.cu
#include <cuda_runtime.h>
#include <unistd.h>

#include <cstdio>
#include <vector>

#include "../paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu"

__global__ void stamp(unsigned long long* t) {
  unsigned long long v;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
  *t = v;
}

int main() {
  const int L = 32;
  struct Case {
    uint64_t chunk;
    int n;
  };
  for (Case cs : {Case{256 << 10, 512}, Case{256 << 10, 3970}, Case{8 << 10, 16384}, Case{8 << 10, 65536},
                  Case{2 << 10, 65536}}) {
    const uint64_t chunk = cs.chunk;
    const int n = cs.n;
    const uint64_t pool_bytes = uint64_t(n) * chunk * L;
    char *pool, *slot, *hostbuf, *dbuf;
    cudaMalloc(&pool, pool_bytes);
    cudaMalloc(&slot, uint64_t(n) * chunk);
    cudaMalloc(&dbuf, 32 << 20);
    cudaHostAlloc(&hostbuf, 32 << 20, 0);
    std::vector<uint64_t> off(n);
    for (int i = 0; i < n; ++i) off[i] = uint64_t((i * 7919) % n) * chunk * L;  // scattered, block-major
    uint64_t* doff;
    cudaMalloc(&doff, n * 8);
    cudaMemcpy(doff, off.data(), n * 8, cudaMemcpyHostToDevice);
    unsigned long long* ts;
    cudaMallocHost(&ts, 64);
    cudaStream_t s, s2;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t a, b, x;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
    aeg::CopyArgs ca;
    ca.src = pool;
    ca.src_off = doff;
    ca.src_lstride = chunk;
    ca.dst = slot;
    ca.chunk = chunk;
    ca.nl = 1;
    ca.n = n;
    const double alg = 2.0 * n * chunk;
    for (int impl : {aeg::IMPL_LSU, aeg::IMPL_BULK, aeg::IMPL_WARP, aeg::IMPL_BULKW}) {
      for (char mode : {'A', 'C'}) {
        double tot = 0, span = 0;
        const int R = 20;
        for (int r = 0; r < R + 2; ++r) {
          if (mode == 'B') {
            cudaStreamSynchronize(s);
            usleep(2000);
          }
          if (mode == 'D') cudaEventRecord(a, s);
          if (mode == 'C' || mode == 'D') {
            cudaMemcpyAsync(hostbuf, dbuf, 32 << 20, cudaMemcpyDeviceToHost, s2);
            cudaEventRecord(x, s2);
            cudaStreamWaitEvent(s, x, 0);
          }
          if (mode != 'D') cudaEventRecord(a, s);
          stamp<<<1, 1, 0, s>>>(ts);
          aeg::launch_copy(ca, impl, 0, s);
          stamp<<<1, 1, 0, s>>>(ts + 1);
          cudaEventRecord(b, s);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (r >= 2) {
            tot += ms;
            span += (ts[1] - ts[0]) * 1e-6;
          }
        }
        printf("chunk=%6llu n=%5d %s %c  event %.1f us (%.0f GB/s)   stamp-to-stamp %.1f us (%.0f GB/s)\n",
               (unsigned long long)chunk, n, impl == aeg::IMPL_LSU ? "LSU " : impl == aeg::IMPL_BULK ? "BULK" : impl == aeg::IMPL_WARP ? "WARP" : "BLKW",
               mode, 1e3 * tot / R, alg / (tot / R) / 1e6, 1e3 * span / R, alg / (span / R) / 1e6);
      }
    }
    cudaFree(pool);
    cudaFree(slot);
    cudaFree(dbuf);
    cudaFreeHost(hostbuf);
  }
  return 0;
}
