// AUTO kernel threshold check: gather (paged -> contiguous, scattered block-major pool) and scatter
// (contiguous -> paged) of ~1 GiB per launch at chunk sizes 16 KiB .. 512 KiB, LSU vs BULK vs WARP,
// event-timed (10 launches after 2 warm-ups).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -o build/threshold_probe tools/threshold_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "../paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu"

int main() {
  const int L = 8;
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (uint64_t chunk : {16ull << 10, 32ull << 10, 64ull << 10, 128ull << 10, 256ull << 10, 512ull << 10}) {
    const int n = int((1ull << 30) / chunk);
    char *pool, *slot;
    cudaMalloc(&pool, uint64_t(n) * chunk * L);
    cudaMalloc(&slot, uint64_t(n) * chunk);
    std::vector<uint64_t> off(n);
    for (int i = 0; i < n; ++i) off[i] = uint64_t((uint64_t(i) * 7919) % n) * chunk * L;
    uint64_t* doff;
    cudaMalloc(&doff, n * 8);
    cudaMemcpy(doff, off.data(), n * 8, cudaMemcpyHostToDevice);
    for (int dir = 0; dir < 2; ++dir) {
      aeg::CopyArgs ca;
      ca.chunk = chunk;
      ca.nl = 1;
      ca.n = n;
      if (dir == 0) {
        ca.src = pool, ca.src_off = doff, ca.src_lstride = chunk, ca.dst = slot;
      } else {
        ca.src = slot, ca.dst = pool, ca.dst_off = doff, ca.dst_lstride = chunk, ca.l_first = 3;
      }
      const double alg = 2.0 * n * chunk;
      for (int impl : {aeg::IMPL_LSU, aeg::IMPL_BULK, aeg::IMPL_WARP}) {
        float tot = 0;
        for (int r = 0; r < 12; ++r) {
          cudaEventRecord(a, s);
          aeg::launch_copy(ca, impl, 0, s);
          cudaEventRecord(b, s);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (r >= 2) tot += ms;
        }
        printf("%s chunk=%4llu KiB n=%6d %s %7.1f us %6.0f GB/s\n", dir ? "scatter" : "gather ",
               (unsigned long long)(chunk >> 10), n,
               impl == aeg::IMPL_LSU ? "LSU " : impl == aeg::IMPL_BULK ? "BULK" : "WARP", 1e3 * tot / 10,
               alg / (tot / 10) / 1e6);
      }
    }
    cudaFree(pool);
    cudaFree(slot);
    cudaFree(doff);
  }
  return 0;
}
