// Is a small zero-copy read of pinned host memory (the block-table fetch kernel's access) starved by
// a concurrent copy-engine H2D stream?  Times a 1-CTA kernel reading `bytes` from mapped pinned
// memory alone, next to a 4 GiB H2D cudaMemcpyAsync, and next to a 4 GiB D2H, and the same read done
// by a tiny cudaMemcpyAsync H2D on another stream.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/zcs tools/zero_copy_starvation_probe.cu
#include <cuda_runtime.h>
#include <unistd.h>

#include <cstdio>
#include <cstdint>

__global__ void fetch(uint2* dst, const uint2* src, uint64_t words) {
  for (uint64_t w = threadIdx.x; w < words; w += blockDim.x) {
    uint2 v;
    asm volatile("ld.global.cv.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(src + w));
    dst[w] = v;
  }
}

int main() {
  const size_t big = 4ull << 30;
  char *hbig, *dbig, *hsmall, *dsmall, *hsmall_dev;
  cudaHostAlloc(&hbig, big, cudaHostAllocPortable);
  cudaMalloc(&dbig, big);
  cudaHostAlloc(&hsmall, 1 << 20, cudaHostAllocMapped);
  cudaHostGetDevicePointer(reinterpret_cast<void**>(&hsmall_dev), hsmall, 0);
  cudaMalloc(&dsmall, 1 << 20);
  cudaStream_t sa, sb;
  cudaStreamCreateWithFlags(&sa, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&sb, cudaStreamNonBlocking);
  cudaEvent_t a0, a1, b0, b1;
  for (cudaEvent_t* e : {&a0, &a1, &b0, &b1}) cudaEventCreate(e);
  for (size_t bytes : {size_t(512), size_t(32768)}) {
    for (int bg = 0; bg < 3; ++bg) {  // 0 none, 1 H2D, 2 D2H in the background
      for (int how = 0; how < 2; ++how) {  // 0 zero-copy kernel, 1 cudaMemcpyAsync
        cudaDeviceSynchronize();
        cudaEventRecord(a0, sa);
        if (bg == 1) cudaMemcpyAsync(dbig, hbig, big, cudaMemcpyHostToDevice, sa);
        if (bg == 2) cudaMemcpyAsync(hbig, dbig, big, cudaMemcpyDeviceToHost, sa);
        cudaEventRecord(a1, sa);
        usleep(5000);  // the background copy is streaming
        cudaEventRecord(b0, sb);
        if (how == 0)
          fetch<<<1, 256, 0, sb>>>(reinterpret_cast<uint2*>(dsmall), reinterpret_cast<const uint2*>(hsmall_dev), bytes / 8);
        else
          cudaMemcpyAsync(dsmall, hsmall, bytes, cudaMemcpyHostToDevice, sb);
        cudaEventRecord(b1, sb);
        cudaDeviceSynchronize();
        float tb, ta;
        cudaEventElapsedTime(&tb, b0, b1);
        cudaEventElapsedTime(&ta, a0, a1);
        printf("read %6zu B by %-14s background %-4s: %9.3f ms (background copy %7.1f ms)\n", bytes,
               how ? "cudaMemcpyAsync" : "zero-copy kernel", bg == 0 ? "none" : bg == 1 ? "H2D" : "D2H", tb, ta);
      }
    }
  }
  return 0;
}
