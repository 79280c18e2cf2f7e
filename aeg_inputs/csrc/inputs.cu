// libaeginputs.so — synthetic input generation and checking for tests and bench.py.
//
// NOT part of the product and holds none of the method's arithmetic: it only evaluates the
// counter-based content generator of aeg_inputs/gen.py (word w of a region with key base K is
// splitmix64(seed ^ (K + w))) at addresses and keys it is given, and provides a synthetic
// per-layer consumer and a delay kernel.  Where to write or expect which key always comes from the
// caller (the oracle's placement), never from libaegkv.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

namespace {

__host__ __device__ __forceinline__ uint64_t sm64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Fill n chunks: chunk i at base + off[i] gets words sm64(seed ^ (key[i] + w)), w < chunk/8.
__global__ void fill_chunks(char* base, const uint64_t* off, const uint64_t* key, uint64_t n, uint64_t chunk,
                            uint64_t seed) {
  const uint64_t wpc = chunk / 8;
  const uint64_t total = n * wpc;
  for (uint64_t t = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; t < total; t += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t i = t / wpc, w = t - i * wpc;
    reinterpret_cast<uint64_t*>(base + off[i])[w] = sm64(seed ^ (key[i] + w));
  }
}

__global__ void verify_chunks(const char* base, const uint64_t* off, const uint64_t* key, uint64_t n, uint64_t chunk,
                              uint64_t seed, unsigned long long* bad, unsigned long long* first) {
  const uint64_t wpc = chunk / 8;
  const uint64_t total = n * wpc;
  unsigned long long mine = 0;
  for (uint64_t t = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; t < total; t += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t i = t / wpc, w = t - i * wpc;
    if (reinterpret_cast<const uint64_t*>(base + off[i])[w] != sm64(seed ^ (key[i] + w))) {
      ++mine;
      atomicMin(first, (unsigned long long)t);
    }
  }
  if (mine) atomicAdd(bad, mine);
}

// Region fill for an arbitrary byte count (tail word truncated little-endian).
__global__ void fill_region(char* p, uint64_t nbytes, uint64_t seed, uint64_t key) {
  const uint64_t nw = nbytes / 8;
  for (uint64_t w = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; w < nw; w += uint64_t(gridDim.x) * blockDim.x)
    reinterpret_cast<uint64_t*>(p)[w] = sm64(seed ^ (key + w));
  if (blockIdx.x == 0 && threadIdx.x == 0 && (nbytes & 7)) {
    const uint64_t v = sm64(seed ^ (key + nw));
    for (uint64_t b = 0; b < (nbytes & 7); ++b) p[nw * 8 + b] = char((v >> (8 * b)) & 0xFF);
  }
}

__global__ void verify_region(const char* p, uint64_t nbytes, uint64_t seed, uint64_t key, unsigned long long* bad,
                              unsigned long long* first) {
  const uint64_t nw = nbytes / 8;
  unsigned long long mine = 0;
  for (uint64_t w = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; w < nw; w += uint64_t(gridDim.x) * blockDim.x)
    if (reinterpret_cast<const uint64_t*>(p)[w] != sm64(seed ^ (key + w))) {
      ++mine;
      atomicMin(first, (unsigned long long)w);
    }
  if (blockIdx.x == 0 && threadIdx.x == 0 && (nbytes & 7)) {
    const uint64_t v = sm64(seed ^ (key + nw));
    for (uint64_t b = 0; b < (nbytes & 7); ++b)
      if ((unsigned char)p[nw * 8 + b] != ((v >> (8 * b)) & 0xFF)) ++mine;
  }
  if (mine) atomicAdd(bad, mine);
}

// Synthetic decode-layer consumer: XOR of every word of n chunks (a stand-in for attention reading
// its KV after aeg_layer_ready); the XOR lands in *out (atomicXor).
__global__ void consume_chunks(const char* base, const uint64_t* off, uint64_t n, uint64_t chunk,
                               unsigned long long* out) {
  const uint64_t vpc = chunk / 16;
  const uint64_t total = n * vpc;
  uint64_t acc = 0;
  for (uint64_t t = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; t < total; t += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t i = t / vpc, v = t - i * vpc;
    const uint4 x = reinterpret_cast<const uint4*>(base + off[i])[v];
    acc ^= (uint64_t(x.y) << 32 | x.x) ^ (uint64_t(x.w) << 32 | x.z);
  }
  for (int s = 16; s > 0; s >>= 1) acc ^= __shfl_xor_sync(0xffffffffu, acc, s);
  if ((threadIdx.x & 31) == 0 && acc) atomicXor(out, (unsigned long long)acc);
}

// Deterministic race-test gate: holds its stream until the host writes a nonzero value into the
// pinned (device-mapped) flag, or at most 60 s (a test that fails while its gate is closed must not
// hang the GPU: the streams behind the gate drain and the test reports a data mismatch instead).
__global__ void gate(const volatile int* flag) {
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    if (*flag != 0) return;
    __nanosleep(1000);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < 60ull * 1000000000ull);
}

// GPU-wide nanosecond clock, comparable across processes sharing the GPU (cross-process timing of
// the host-route hand-off, where CUDA events cannot be shared with timing enabled).
__global__ void stamp(unsigned long long* out) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  *out = t;
}

__global__ void spin(long long cycles) {
  const long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}

int grid_for(uint64_t work) {
  uint64_t g = (work + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  if (g < 1) g = 1;
  return int(g);
}

struct DevTables {
  uint64_t* d = nullptr;
  cudaError_t e = cudaSuccess;
  DevTables(const uint64_t* a, const uint64_t* b, uint64_t n, cudaStream_t s) {
    e = cudaMallocAsync(&d, 2 * n * 8 + 16, s);
    if (e != cudaSuccess) return;
    if (n) e = cudaMemcpyAsync(d, a, n * 8, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && b && n) e = cudaMemcpyAsync(d + n, b, n * 8, cudaMemcpyHostToDevice, s);
  }
  void release(cudaStream_t s) {
    if (d) cudaFreeAsync(d, s);
  }
};

}  // namespace

extern "C" {

int aegin_fill_chunks(void* base, const uint64_t* off, const uint64_t* key, uint64_t n, uint64_t chunk, uint64_t seed,
                      void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (n == 0) return 0;
  DevTables t(off, key, n, s);
  if (t.e != cudaSuccess) return int(t.e);
  fill_chunks<<<grid_for(n * chunk / 8), 256, 0, s>>>(static_cast<char*>(base), t.d, t.d + n, n, chunk, seed);
  cudaError_t e = cudaGetLastError();
  t.release(s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  return int(e);
}

int aegin_verify_chunks(const void* base, const uint64_t* off, const uint64_t* key, uint64_t n, uint64_t chunk,
                        uint64_t seed, uint64_t* bad, uint64_t* first, void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  *bad = 0;
  *first = ~0ull;
  if (n == 0) return 0;
  DevTables t(off, key, n, s);
  if (t.e != cudaSuccess) return int(t.e);
  unsigned long long* r;
  cudaError_t e = cudaMallocAsync(&r, 16, s);
  if (e != cudaSuccess) return int(e);
  unsigned long long init[2] = {0, ~0ull};
  cudaMemcpyAsync(r, init, 16, cudaMemcpyHostToDevice, s);
  verify_chunks<<<grid_for(n * chunk / 8), 256, 0, s>>>(static_cast<const char*>(base), t.d, t.d + n, n, chunk, seed, r,
                                                        r + 1);
  e = cudaGetLastError();
  unsigned long long out[2] = {0, 0};
  if (e == cudaSuccess) e = cudaMemcpyAsync(out, r, 16, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(r, s);
  t.release(s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  *bad = out[0];
  *first = out[1];
  return int(e);
}

int aegin_fill_region(void* p, uint64_t nbytes, uint64_t seed, uint64_t key, void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (!nbytes) return 0;
  fill_region<<<grid_for(nbytes / 8 + 1), 256, 0, s>>>(static_cast<char*>(p), nbytes, seed, key);
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  return int(e);
}

int aegin_verify_region(const void* p, uint64_t nbytes, uint64_t seed, uint64_t key, uint64_t* bad, uint64_t* first,
                        void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  *bad = 0;
  *first = ~0ull;
  if (!nbytes) return 0;
  unsigned long long* r;
  cudaError_t e = cudaMallocAsync(&r, 16, s);
  if (e != cudaSuccess) return int(e);
  unsigned long long init[2] = {0, ~0ull};
  cudaMemcpyAsync(r, init, 16, cudaMemcpyHostToDevice, s);
  verify_region<<<grid_for(nbytes / 8 + 1), 256, 0, s>>>(static_cast<const char*>(p), nbytes, seed, key, r, r + 1);
  e = cudaGetLastError();
  unsigned long long out[2] = {0, 0};
  if (e == cudaSuccess) e = cudaMemcpyAsync(out, r, 16, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(r, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  *bad = out[0];
  *first = out[1];
  return int(e);
}

// Enqueue a consumer of n chunks on `stream` (no synchronisation); `dev_off` is a DEVICE array and
// `out` a device (or mapped host) u64 that receives the XOR.  Returns the launch error.
int aegin_consume(const void* base, const uint64_t* dev_off, uint64_t n, uint64_t chunk, void* out, void* stream) {
  if (!n) return 0;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  consume_chunks<<<grid_for(n * chunk / 16), 256, 0, s>>>(static_cast<const char*>(base), dev_off, n, chunk,
                                                          static_cast<unsigned long long*>(out));
  return int(cudaGetLastError());
}

// Plain copy between any two pointers (device, pinned or pageable host) for test read-back.
int aegin_copy(void* dst, const void* src, uint64_t n) { return int(cudaMemcpy(dst, src, n, cudaMemcpyDefault)); }

int aegin_sync(void) { return int(cudaDeviceSynchronize()); }

// Baseline for the bench (what the paper's "memcpy(async)" per block amounts to for paged KV): one
// cudaMemcpyAsync per chunk, dst_base + dst_off[i] <- src_base + src_off[i], on `stream`
// (copy engines; host or device pointers, UVA).
int aegin_copy_chunks(void* dst_base, const uint64_t* dst_off, const void* src_base, const uint64_t* src_off,
                      uint64_t n, uint64_t chunk, void* stream) {
  for (uint64_t i = 0; i < n; ++i) {
    cudaError_t e = cudaMemcpyAsync(static_cast<char*>(dst_base) + dst_off[i],
                                    static_cast<const char*>(src_base) + src_off[i], chunk, cudaMemcpyDefault,
                                    static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return int(e);
  }
  return 0;
}

// Load every kernel of this library now (no lazy module load later, which would wait for a
// running gate kernel and deadlock a race test).
int aegin_preload(void) {
  cudaFuncAttributes a;
  cudaError_t e = cudaFuncGetAttributes(&a, fill_chunks);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, verify_chunks);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, fill_region);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, verify_region);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, consume_chunks);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, gate);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, spin);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, stamp);
  return int(e);
}

int aegin_gate(const void* pinned_flag, void* stream) {
  gate<<<1, 1, 0, static_cast<cudaStream_t>(stream)>>>(static_cast<const volatile int*>(pinned_flag));
  return int(cudaGetLastError());
}

int aegin_stamp(void* dev_u64, void* stream) {
  stamp<<<1, 1, 0, static_cast<cudaStream_t>(stream)>>>(static_cast<unsigned long long*>(dev_u64));
  return int(cudaGetLastError());
}

int aegin_spin(long long cycles, void* stream) {
  spin<<<1, 1, 0, static_cast<cudaStream_t>(stream)>>>(cycles);
  return int(cudaGetLastError());
}

// Host-side multi-threaded fill of pageable memory (Model Cache content): same generator.
int aegin_host_fill(void* p, uint64_t nbytes, uint64_t seed, uint64_t key, int threads) {
  if (threads < 1) threads = 1;
  const uint64_t nw = nbytes / 8;
  std::vector<std::thread> ts;
  for (int t = 0; t < threads; ++t)
    ts.emplace_back([=] {
      const uint64_t a = nw * t / threads, b = nw * (t + 1) / threads;
      uint64_t* q = static_cast<uint64_t*>(p);
      for (uint64_t w = a; w < b; ++w) q[w] = sm64(seed ^ (key + w));
    });
  for (auto& t : ts) t.join();
  if (nbytes & 7) {
    const uint64_t v = sm64(seed ^ (key + nw));
    for (uint64_t b = 0; b < (nbytes & 7); ++b) static_cast<char*>(p)[nw * 8 + b] = char((v >> (8 * b)) & 0xFF);
  }
  return 0;
}

// Strided variant: `rows` runs of `width` bytes at a `pitch`, run r starting at p + r * pitch; every
// word holds the value it has in the dense fill of the whole [rows x pitch] region with base `key`,
// so a run is bit-identical to the same bytes of a dense fill (used to materialise only one TP
// rank's column slice of a row-major tensor in a sparse Model Cache).  pitch, width multiples of 8.
int aegin_host_fill_2d(void* p, uint64_t rows, uint64_t pitch, uint64_t width, uint64_t seed, uint64_t key,
                       int threads) {
  if ((pitch & 7) || (width & 7) || width > pitch) return 1;
  if (threads < 1) threads = 1;
  std::vector<std::thread> ts;
  for (int t = 0; t < threads; ++t)
    ts.emplace_back([=] {
      for (uint64_t r = rows * t / threads; r < rows * (t + 1) / threads; ++r) {
        uint64_t* q = reinterpret_cast<uint64_t*>(static_cast<char*>(p) + r * pitch);
        const uint64_t w0 = r * pitch / 8;
        for (uint64_t w = 0; w < width / 8; ++w) q[w] = sm64(seed ^ (key + w0 + w));
      }
    });
  for (auto& t : ts) t.join();
  return 0;
}

}  // extern "C"
