// IPC event semantics probe.  Parent: spin kernel (~1 s) then a flag write then cudaEventRecord on an
// interprocess event; the handle goes to a forked child through a pipe.  Child: opens the handle and
// reports (a) cudaEventQuery right away, (b) how long cudaEventSynchronize blocks, (c) whether a
// kernel launched after cudaStreamWaitEvent sees the flag.  Build: nvcc -O2 -o build/ipc_probe tools/ipc_probe.cu
#include <cuda_runtime.h>
#include <sys/wait.h>
#include <unistd.h>

#include <chrono>
#include <cstdio>

__global__ void spin(long long c) {
  long long t = clock64();
  while (clock64() - t < c) {
  }
}
__global__ void setf(int* f) { *(volatile int*)f = 1; }
__global__ void readf(int* f, int* out) { *out = *(volatile int*)f; }

struct Msg {
  cudaIpcEventHandle_t ev;
  cudaIpcMemHandle_t mem;
};

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  int p2c[2], c2p[2];
  if (pipe(p2c) || pipe(c2p)) return 1;
  pid_t pid = fork();
  if (pid == 0) {  // child
    Msg m;
    if (read(p2c[0], &m, sizeof m) != sizeof m) return 2;
    cudaEvent_t e;
    cudaError_t r = cudaIpcOpenEventHandle(&e, m.ev);
    printf("child: open event: %s\n", cudaGetErrorString(r));
    int* f;
    r = cudaIpcOpenMemHandle((void**)&f, m.mem, cudaIpcMemLazyEnablePeerAccess);
    printf("child: open mem: %s\n", cudaGetErrorString(r));
    char go = 1;
    write(c2p[1], &go, 1);  // parent records only now
    char rec;
    read(p2c[0], &rec, 1);
    double t0 = now();
    printf("child: query right after parent's record: %s\n", cudaGetErrorString(cudaEventQuery(e)));
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    int* out;
    cudaMallocHost(&out, 4);
    *out = -1;
    cudaStreamWaitEvent(s, e, 0);
    readf<<<1, 1, 0, s>>>(f, out);
    cudaStreamSynchronize(s);
    printf("child: kernel after cudaStreamWaitEvent saw flag=%d after %.3f s\n", *out, now() - t0);
    double t1 = now();
    cudaEventSynchronize(e);
    printf("child: cudaEventSynchronize returned after %.3f s, query now: %s\n", now() - t1,
           cudaGetErrorString(cudaEventQuery(e)));
    return 0;
  }
  // parent
  cudaFree(0);
  cudaEvent_t e;
  cudaEventCreateWithFlags(&e, cudaEventDisableTiming | cudaEventInterprocess);
  int* f;
  cudaMalloc(&f, 4);
  cudaMemset(f, 0, 4);
  cudaDeviceSynchronize();
  Msg m;
  cudaIpcGetEventHandle(&m.ev, e);
  cudaIpcGetMemHandle(&m.mem, f);
  write(p2c[1], &m, sizeof m);
  char go;
  read(c2p[0], &go, 1);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  spin<<<1, 1, 0, s>>>(2000000000LL);  // ~1 s
  setf<<<1, 1, 0, s>>>(f);
  cudaEventRecord(e, s);
  printf("parent: recorded behind a ~1 s spin; local query: %s\n", cudaGetErrorString(cudaEventQuery(e)));
  fflush(stdout);
  char rec = 1;
  write(p2c[1], &rec, 1);
  int st;
  waitpid(pid, &st, 0);
  cudaDeviceSynchronize();
  return 0;
}
