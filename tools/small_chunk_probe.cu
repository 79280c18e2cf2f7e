// Small-chunk gather/scatter probe: event-timed back-to-back launches of the product
// copy kernels (csrc/kernels/copy.cu, included verbatim; BULKW geometry set by -D) on scattered
// block tables, for 2-32 KiB chunks, gather (paged -> contiguous) and scatter (contiguous -> paged).
// GB/s = algorithmic bytes (2 x payload) / median event time.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DAEG_BW_WARPS=4 -DAEG_BW_SMEM_KIB=192 \
//          -o build/small_chunk_probe tools/small_chunk_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstdio>
#include <vector>

#include "../paper_conf_sosp_xiang0qyzyzl0025_b200/csrc/kernels/copy.cu"

int main() {
  const uint64_t payload = 1ull << 30;  // 1 GiB per launch each way
  const bool mig = getenv("MIGRATE") != nullptr;  // paged -> paged (H5 local) at large chunks
  std::vector<uint64_t> chunks = {2048ull, 4096ull, 8192ull, 16384ull, 32768ull};
  if (mig) chunks = {32768ull, 262144ull, 327680ull};
  if (getenv("CHUNKS")) {  // comma-separated override
    chunks.clear();
    for (char* p = getenv("CHUNKS"); *p;) {
      chunks.push_back(strtoull(p, &p, 10));
      if (*p == ',') ++p;
    }
  }
  for (uint64_t chunk : chunks) {
    const int n = int(payload / chunk);
    char *pool, *slot;
    // blocks scattered over SPREAD x the payload (default 2; SPREAD=30 mimics 30 GB pools)
    const uint64_t spread = getenv("SPREAD") ? strtoull(getenv("SPREAD"), nullptr, 10) : 2;
    cudaMalloc(&pool, spread * payload);
    cudaMalloc(&slot, payload);
    std::vector<uint64_t> off(n);
    for (int i = 0; i < n; ++i) off[i] = uint64_t((uint64_t(i) * 7919) % (spread * n)) * chunk;
    std::sort(off.begin(), off.end());
    off.erase(std::unique(off.begin(), off.end()), off.end());
    while (int(off.size()) < n) off.push_back(off.back() + chunk);
    for (int i = n - 1; i > 0; --i) std::swap(off[i], off[(uint64_t(i) * 2654435761u) % (i + 1)]);
    uint64_t* doff;
    cudaMalloc(&doff, n * 8);
    cudaMemcpy(doff, off.data(), n * 8, cudaMemcpyHostToDevice);
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    uint64_t* doff2 = nullptr;
    char* pool2 = nullptr;
    if (mig) {  // a second scattered table into a second pool
      std::vector<uint64_t> off2(off);
      for (int i = n - 1; i > 0; --i) std::swap(off2[i], off2[(uint64_t(i) * 40503u + 7) % (i + 1)]);
      cudaMalloc(&doff2, n * 8);
      cudaMemcpy(doff2, off2.data(), n * 8, cudaMemcpyHostToDevice);
      cudaMalloc(&pool2, spread * payload);
    }
    for (int dir = 0; dir < (mig ? 1 : 2); ++dir) {
      aeg::CopyArgs ca;
      if (mig) {
        ca.src = pool;
        ca.src_off = doff;
        ca.dst = pool2;
        ca.dst_off = doff2;
      } else if (dir == 0) {
        ca.src = pool;
        ca.src_off = doff;
        ca.dst = slot;
      } else {
        ca.src = slot;
        ca.dst = pool;
        ca.dst_off = doff;
      }
      ca.src_lstride = ca.dst_lstride = chunk;
      ca.chunk = chunk;
      ca.nl = 1;
      ca.n = n;
      if (getenv("SWEEP")) {  // BULKW with explicit piece sizes (>= 2 stages per warp)
        using namespace aeg;
        auto kern = mig ? copy_bulkw<true, true> : dir == 0 ? copy_bulkw<true, false> : copy_bulkw<false, true>;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kBwSmem);
        std::vector<uint64_t> pieces = {chunk, 16384, 12288, 10240, 8192, 6144, 5120, 4096, 2048};
        std::sort(pieces.begin(), pieces.end());
        pieces.erase(std::unique(pieces.begin(), pieces.end()), pieces.end());
        for (uint64_t piece : pieces) {
          if (piece > chunk || piece * 2 > uint64_t(kBwSmem / kBwWarps)) continue;
          const uint64_t items = uint64_t(n) * ((chunk + piece - 1) / piece);
          int occ = 0;
          cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBwWarps * 32, kBwSmem);
          // CTAS_PER_SM caps the grid below the occupancy limit (in-flight bulk copies per SM)
          const int cps = getenv("CTAS_PER_SM") ? atoi(getenv("CTAS_PER_SM")) : occ;
          uint64_t grid = uint64_t(148) * std::max(1, std::min(occ, cps));
          if (grid > (items + kBwWarps - 1) / kBwWarps) grid = (items + kBwWarps - 1) / kBwWarps;
          std::vector<float> ts;
          for (int r = 0; r < 12; ++r) {
            cudaEventRecord(a, s);
            kern<<<unsigned(grid), kBwWarps * 32, kBwSmem, s>>>(ca, uint32_t(piece));
            cudaEventRecord(b, s);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (r >= 2) ts.push_back(ms);
          }
          std::sort(ts.begin(), ts.end());
          const double med = ts[ts.size() / 2];
          printf("chunk=%6llu %s BULKW warps=%d smem=%dK ctas/SM=%d piece=%6llu median %8.1f us  %7.0f GB/s\n",
                 (unsigned long long)chunk, mig ? "migrate" : dir ? "scatter" : "gather ", kBwWarps, kBwSmem >> 10,
                 int(grid / 148),
                 (unsigned long long)piece, med * 1e3, 2.0 * payload / (med * 1e6));
        }
        continue;
      }
      for (int impl : {aeg::IMPL_LSU, aeg::IMPL_WARP, aeg::IMPL_BULK, aeg::IMPL_BULKW}) {
        std::vector<float> ts;
        for (int r = 0; r < 12; ++r) {
          cudaEventRecord(a, s);
          cudaError_t e = aeg::launch_copy(ca, impl, 0, s);
          cudaEventRecord(b, s);
          cudaEventSynchronize(b);
          if (e != cudaSuccess || cudaGetLastError() != cudaSuccess) {
            printf("error %s\n", cudaGetErrorString(e));
            return 1;
          }
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (r >= 2) ts.push_back(ms);
        }
        std::sort(ts.begin(), ts.end());
        const double med = ts[ts.size() / 2];
        printf("chunk=%6llu %s %-5s median %8.1f us  %7.0f GB/s (best %7.0f)\n", (unsigned long long)chunk,
               dir ? "scatter" : "gather ",
               impl == aeg::IMPL_LSU ? "LSU" : impl == aeg::IMPL_WARP ? "WARP" : impl == aeg::IMPL_BULK ? "BULK" : "BULKW",
               med * 1e3, 2.0 * payload / (med * 1e6), 2.0 * payload / (ts[0] * 1e6));
      }
    }
    cudaFree(pool);
    cudaFree(slot);
    cudaFree(doff);
    if (mig) {
      cudaFree(pool2);
      cudaFree(doff2);
    }
  }
  return 0;
}
