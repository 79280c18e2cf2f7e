// N2: why does P->C into the node-shared CPU KV cache run at 46-50 GB/s while the
// private pinned pool gets 54-57?  Times 1 GiB D2H / H2D cudaMemcpyAsync into host memory obtained
// several ways, all page-locked with cudaHostRegister (Portable | Mapped) except cudaHostAlloc:
//   hostalloc  cudaHostAlloc
//   anon_thp   anonymous mmap + MADV_HUGEPAGE, first touch, register (the private pool's path)
//   shm        POSIX shm_open + mmap MAP_SHARED (4 KiB pages), first touch, register (current N2 path)
//   shm_thp    same + MADV_HUGEPAGE (effective only if shmem THP is enabled on the host)
//   shm_popul  same + MAP_POPULATE
//   memfd_huge memfd_create(MFD_HUGETLB) (needs reserved huge pages)
// Build: nvcc -O2 -o /tmp/shm_probe tools/shm_probe.cu
#include <cuda_runtime.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <unistd.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#ifndef MFD_HUGETLB
#define MFD_HUGETLB 0x0004U
#endif

static void touch(char* p, size_t n) {
  std::vector<std::thread> ts;
  for (int t = 0; t < 16; ++t)
    ts.emplace_back([=] {
      for (size_t o = n * t / 16; o < n * (t + 1) / 16; o += 4096) p[o] = 1;
    });
  for (auto& t : ts) t.join();
}

int main() {
  const size_t n = 1ull << 30;
  char* dbuf;
  cudaMalloc(&dbuf, n);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (const char* kind : {"hostalloc", "anon_thp", "shm", "shm_thp", "shm_popul", "memfd_huge"}) {
    char* h = nullptr;
    std::string k = kind;
    bool reg = true;
    if (k == "hostalloc") {
      if (cudaHostAlloc(&h, n, cudaHostAllocPortable) != cudaSuccess) h = nullptr;
      reg = false;
    } else if (k == "anon_thp") {
      void* p = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
      if (p != MAP_FAILED) {
        madvise(p, n, MADV_HUGEPAGE);
        h = static_cast<char*>(p);
      }
    } else if (k == "memfd_huge") {
      int fd = int(syscall(319 /* memfd_create */, "aeg_probe", MFD_HUGETLB));
      if (fd >= 0 && ftruncate(fd, off_t(n)) == 0) {
        void* p = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
        if (p != MAP_FAILED) h = static_cast<char*>(p);
      }
      if (fd >= 0) close(fd);
    } else {
      std::string nm = "/aeg_probe_" + std::to_string(getpid()) + k;
      int fd = shm_open(nm.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
      if (fd >= 0 && ftruncate(fd, off_t(n)) == 0) {
        void* p = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_SHARED | (k == "shm_popul" ? MAP_POPULATE : 0), fd, 0);
        if (p != MAP_FAILED) {
          if (k == "shm_thp") madvise(p, n, MADV_HUGEPAGE);
          h = static_cast<char*>(p);
        }
      }
      if (fd >= 0) close(fd);
      shm_unlink(nm.c_str());
    }
    if (!h) {
      printf("%-11s unavailable\n", kind);
      continue;
    }
    touch(h, n);
    if (reg && cudaHostRegister(h, n, cudaHostRegisterPortable | cudaHostRegisterMapped) != cudaSuccess) {
      printf("%-11s register failed: %s\n", kind, cudaGetErrorString(cudaGetLastError()));
      continue;
    }
    for (int dir = 0; dir < 2; ++dir) {
      std::vector<float> ts;
      for (int r = 0; r < 6; ++r) {
        cudaEventRecord(a, s);
        if (dir == 0)
          cudaMemcpyAsync(h, dbuf, n, cudaMemcpyDeviceToHost, s);
        else
          cudaMemcpyAsync(dbuf, h, n, cudaMemcpyHostToDevice, s);
        cudaEventRecord(b, s);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r) ts.push_back(ms);
      }
      std::sort(ts.begin(), ts.end());
      printf("%-11s %s median %.1f GB/s best %.1f\n", kind, dir ? "H2D" : "D2H", n / (ts[ts.size() / 2] * 1e6),
             n / (ts[0] * 1e6));
    }
    // hugepage share of the mapping (AnonHugePages / ShmemPmdMapped via smaps of this range)
    FILE* f = fopen("/proc/self/smaps", "r");
    char line[512];
    bool in = false;
    while (f && fgets(line, sizeof line, f)) {
      unsigned long lo, hi;
      if (sscanf(line, "%lx-%lx", &lo, &hi) == 2 && strchr(line, ' ') && line[8] != ' ') in = (char*)lo == h;
      if (in && (strstr(line, "AnonHugePages") || strstr(line, "ShmemPmdMapped") || strstr(line, "KernelPageSize")))
        printf("   %s", line);
    }
    if (f) fclose(f);
    if (reg) cudaHostUnregister(h);
    if (k == "hostalloc")
      cudaFreeHost(h);
    else
      munmap(h, n);
  }
  return 0;
}
