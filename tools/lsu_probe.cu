// LSU copy-kernel variants on the configs[2] migrate shape (paged -> paged, 2,346 Llama-2-13B
// blocks x 320 KiB per layer, source layer-major, destination block-major, ~30 GB per side) and on
// the C2 gather shape (3,970 x 256 KiB paged -> contiguous): threads per CTA x 16-byte vectors in
// flight per thread, grid = resident CTAs x 148.  Event-timed, 10 launches after 2 warm-ups.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -o build/lsu_probe tools/lsu_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "../paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu"

namespace {
template <bool SP, bool DP, int T, int U>
__global__ void __launch_bounds__(T) lsu_v(const aeg::CopyArgs a) {
  constexpr uint64_t piece = uint64_t(T) * 16 * U;
  const uint64_t ppc = (a.chunk + piece - 1) / piece;
  const uint64_t items = uint64_t(a.nl) * uint64_t(a.n) * ppc;
  for (uint64_t w = blockIdx.x; w < items; w += gridDim.x) {
    const uint64_t c = w / ppc;
    const uint64_t base = (w - c * ppc) * piece;
    const char* s;
    char* d;
    aeg::item_ptrs<SP, DP>(a, c, s, d);
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t o = base + (uint64_t(u) * T + threadIdx.x) * 16;
      if (o < a.chunk) v[u] = aeg::ld_stream(s + o);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t o = base + (uint64_t(u) * T + threadIdx.x) * 16;
      if (o < a.chunk) aeg::st_stream(d + o, v[u]);
    }
  }
}

template <bool SP, bool DP, int T, int U>
void run(const char* name, const aeg::CopyArgs& a, cudaStream_t s, double alg) {
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, lsu_v<SP, DP, T, U>, T, 0);
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, lsu_v<SP, DP, T, U>);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int cap : {0, 4}) {
    const int ctas = 148 * (cap && per_sm > cap ? cap : per_sm);
    float tot = 0;
    for (int r = 0; r < 12; ++r) {
      cudaEventRecord(e0, s);
      lsu_v<SP, DP, T, U><<<ctas, T, 0, s>>>(a);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (r >= 2) tot += ms;
    }
    printf("%-8s T=%4d U=%2d regs=%3d ctas/SM=%d grid=%5d  %7.1f us  %6.0f GB/s\n", name, T, U, fa.numRegs,
           ctas / 148, ctas, 1e3 * tot / 10, alg / (tot / 10) / 1e6);
  }
}
}  // namespace

int main() {
  {  // migrate shape
    const int L = 40, n = 2346;
    const uint64_t chunk = 320 << 10, block = chunk * L;
    const uint64_t slab = (1ull << 30) + (256ull << 20), k = slab / block, nslab = (n + k - 1) / k + 1;
    char *src, *dst;
    cudaMalloc(&src, nslab * slab);
    cudaMalloc(&dst, nslab * slab);
    std::vector<uint64_t> off(2 * n);
    for (int i = 0; i < n; ++i) {
      off[i] = (i / k) * slab + (i % k) * chunk;      // layer-major slab: layer-0 offset, lstride k*chunk
      off[n + i] = (i / k) * slab + (i % k) * block;  // block-major slab: lstride chunk
    }
    uint64_t* doff;
    cudaMalloc(&doff, 2 * n * 8);
    cudaMemcpy(doff, off.data(), 2 * n * 8, cudaMemcpyHostToDevice);
    aeg::CopyArgs a;
    a.src = src;
    a.dst = dst;
    a.src_off = doff;
    a.dst_off = doff + n;
    a.src_lstride = k * chunk;
    a.dst_lstride = chunk;
    a.chunk = chunk;
    a.nl = 1;
    a.n = n;
    a.l_first = 7;
    cudaStream_t s;
    cudaStreamCreate(&s);
    const double alg = 2.0 * n * chunk;
    run<true, true, 256, 8>("migrate", a, s, alg);
    run<true, true, 256, 16>("migrate", a, s, alg);
    run<true, true, 512, 8>("migrate", a, s, alg);
    run<true, true, 128, 16>("migrate", a, s, alg);
    run<true, true, 128, 32>("migrate", a, s, alg);
    run<true, true, 1024, 4>("migrate", a, s, alg);
    cudaFree(src);
    cudaFree(dst);
    cudaFree(doff);
  }
  {  // gather shape
    const int L = 32, n = 3970;
    const uint64_t chunk = 256 << 10;
    char *pool, *slot;
    cudaMalloc(&pool, uint64_t(n) * chunk * L);
    cudaMalloc(&slot, uint64_t(n) * chunk);
    std::vector<uint64_t> off(n);
    for (int i = 0; i < n; ++i) off[i] = uint64_t((i * 7919) % n) * chunk * L;
    uint64_t* doff;
    cudaMalloc(&doff, n * 8);
    cudaMemcpy(doff, off.data(), n * 8, cudaMemcpyHostToDevice);
    aeg::CopyArgs a;
    a.src = pool;
    a.src_off = doff;
    a.src_lstride = chunk;
    a.dst = slot;
    a.chunk = chunk;
    a.nl = 1;
    a.n = n;
    cudaStream_t s;
    cudaStreamCreate(&s);
    const double alg = 2.0 * n * chunk;
    run<true, false, 256, 8>("gather", a, s, alg);
    run<true, false, 256, 16>("gather", a, s, alg);
    run<true, false, 512, 8>("gather", a, s, alg);
    run<true, false, 128, 32>("gather", a, s, alg);
  }
  return 0;
}
