// Why is the in-step gather slower than the same launch alone (bench roofline 0.87-0.90 vs ncu's
// cold 316 us)?  Times one full-size C2 gather launch (3,970 x 256 KiB chunks from a scattered
// block-major pool into a contiguous slot, BULK and LSU) with CUDA events while other traffic of
// the swap step runs on other streams: a 1 GiB D2H, a 1 GiB H2D, both, a concurrent scatter-sized
// copy kernel.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -o build/contention_probe tools/contention_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "../paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu"

int main() {
  const int L = 32, n = 3970;
  const uint64_t chunk = 256 << 10, G = 1ull << 30;
  const uint64_t pool_bytes = uint64_t(n) * chunk * L;
  char *pool, *slot, *slot2, *dbuf, *hbuf;
  cudaMalloc(&pool, pool_bytes);
  cudaMalloc(&slot, uint64_t(n) * chunk);
  cudaMalloc(&slot2, uint64_t(n) * chunk);
  cudaMalloc(&dbuf, G);
  cudaHostAlloc(&hbuf, G, 0);
  std::vector<uint64_t> off(n);
  for (int i = 0; i < n; ++i) off[i] = uint64_t((i * 7919) % n) * chunk * L;
  uint64_t* doff;
  cudaMalloc(&doff, n * 8);
  cudaMemcpy(doff, off.data(), n * 8, cudaMemcpyHostToDevice);
  cudaStream_t s, sd, sh, sk;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&sd, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&sh, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&sk, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  aeg::CopyArgs ga;
  ga.src = pool;
  ga.src_off = doff;
  ga.src_lstride = chunk;
  ga.dst = slot;
  ga.chunk = chunk;
  ga.nl = 1;
  ga.n = n;
  aeg::CopyArgs sa = ga;  // scatter-shaped: contiguous slot2 -> paged pool (layer 1)
  sa.src = slot2;
  sa.src_off = nullptr;
  sa.dst = pool;
  sa.dst_off = doff;
  sa.dst_lstride = chunk;
  sa.l_first = 1;
  const double alg = 2.0 * n * chunk;
  const char* names[] = {"alone", "+D2H 1GiB", "+H2D 1GiB", "+D2H+H2D", "+scatter kernel", "+scatter+D2H+H2D"};
  for (int impl : {aeg::IMPL_BULK, aeg::IMPL_LSU})
    for (int mode = 0; mode < 6; ++mode) {
      double tot = 0;
      const int R = 10;
      for (int r = 0; r < R + 2; ++r) {
        cudaDeviceSynchronize();
        if (mode == 1 || mode == 3 || mode == 5) cudaMemcpyAsync(hbuf, dbuf, G, cudaMemcpyDeviceToHost, sd);
        if (mode == 2 || mode == 3 || mode == 5) cudaMemcpyAsync(dbuf, hbuf, G, cudaMemcpyHostToDevice, sh);
        if (mode == 4 || mode == 5) aeg::launch_copy(sa, impl, 0, sk);
        cudaEventRecord(a, s);
        aeg::launch_copy(ga, impl, 0, s);
        cudaEventRecord(b, s);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r >= 2) tot += ms;
      }
      cudaDeviceSynchronize();
      printf("%s gather %-18s event %.1f us (%.0f GB/s)\n", impl == aeg::IMPL_BULK ? "BULK" : "LSU ", names[mode],
             1e3 * tot / R, alg / (tot / R) / 1e6);
    }
  return 0;
}
