// Block-table copy kernels for B200 (sm_100a).  See copy.h for the addressing contract.
//
// Two implementations of the same byte copy, selected by measurement:
//  * LSU  : 256-thread CTAs; a work item is a 32 KiB piece of one (block, layer) chunk; each
//           thread issues 8 independent 16-byte ld.global.nc.L1::no_allocate (all loads first,
//           then all stores) so ~128 KiB per SM are in flight; the block-table entry of an item
//           is one broadcast load per warp.
//  * BULK : the Blackwell async path: one thread per CTA drives a STAGES-deep ring of PIECE-byte
//           shared-memory buffers with cp.async.bulk (global->smem, mbarrier complete_tx) and
//           cp.async.bulk (smem->global, bulk_group); no data passes through registers.
// Both are persistent: the grid is one wave (148 SMs x resident CTAs) striding over items.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdint>

#include "copy.h"

namespace aeg {
namespace {

constexpr int kSMs = 148;

__device__ __forceinline__ uint4 ld_stream(const void* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

__device__ __forceinline__ void st_stream(void* p, const uint4& v) {
  asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

template <bool SP, bool DP>
__device__ __forceinline__ void item_ptrs(const CopyArgs& a, uint64_t c, const char*& s, char*& d) {
  const uint32_t t = uint32_t(c / uint64_t(a.n));
  const uint32_t i = uint32_t(c - uint64_t(t) * a.n);
  if (SP)
    s = a.src + __ldg(a.src_off + i) + uint64_t(a.l_first + t) * a.src_lstride;
  else
    s = a.src + c * a.chunk;  // (t * n + i) * chunk
  if (DP)
    d = a.dst + __ldg(a.dst_off + i) + uint64_t(a.l_first + t) * a.dst_lstride;
  else
    d = a.dst + c * a.chunk;
}

// ------------------------------------------------------------------------------------- LSU
constexpr int kLsuThreads = 256;
constexpr int kLsuUnroll = 8;
constexpr uint64_t kLsuPiece = uint64_t(kLsuThreads) * 16 * kLsuUnroll;  // 32 KiB

template <bool SP, bool DP>
__global__ void __launch_bounds__(kLsuThreads) copy_lsu(const CopyArgs a) {
  const uint64_t ppc = (a.chunk + kLsuPiece - 1) / kLsuPiece;
  const uint64_t items = uint64_t(a.nl) * uint64_t(a.n) * ppc;
  for (uint64_t w = blockIdx.x; w < items; w += gridDim.x) {
    const uint64_t c = w / ppc;
    const uint64_t base = (w - c * ppc) * kLsuPiece;
    const char* s;
    char* d;
    item_ptrs<SP, DP>(a, c, s, d);
    uint4 v[kLsuUnroll];
    if (base + kLsuPiece <= a.chunk) {
#pragma unroll
      for (int u = 0; u < kLsuUnroll; ++u) v[u] = ld_stream(s + base + (uint64_t(u) * kLsuThreads + threadIdx.x) * 16);
#pragma unroll
      for (int u = 0; u < kLsuUnroll; ++u) st_stream(d + base + (uint64_t(u) * kLsuThreads + threadIdx.x) * 16, v[u]);
    } else {
#pragma unroll
      for (int u = 0; u < kLsuUnroll; ++u) {
        const uint64_t o = base + (uint64_t(u) * kLsuThreads + threadIdx.x) * 16;
        if (o < a.chunk) v[u] = ld_stream(s + o);
      }
#pragma unroll
      for (int u = 0; u < kLsuUnroll; ++u) {
        const uint64_t o = base + (uint64_t(u) * kLsuThreads + threadIdx.x) * 16;
        if (o < a.chunk) st_stream(d + o, v[u]);
      }
    }
  }
}

// ------------------------------------------------------------------------------------ WARP
// Small chunks (<= 8 KiB, e.g. TP-sharded GQA caches with one KV head per rank): a warp takes 32
// consecutive chunks, each lane resolves one chunk's pointers (one coalesced block-table load per
// 32 chunks), and the warp then copies the chunks one after another with the pointers broadcast by
// __shfl_sync — the north star's warp-level index broadcast.
constexpr int kWarpThreads = 256;
constexpr int kWarpUnroll = 4;

template <bool SP, bool DP>
__global__ void __launch_bounds__(kWarpThreads) copy_warp(const CopyArgs a) {
  const uint64_t total = uint64_t(a.nl) * uint64_t(a.n);
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (uint64_t(blockIdx.x) * kWarpThreads + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * kWarpThreads) >> 5;
  const uint32_t vecs = uint32_t(a.chunk / 16);
  for (uint64_t g = warp * 32; g < total; g += nwarps * 32) {
    const uint64_t c = g + lane;
    const char* s = nullptr;
    char* d = nullptr;
    if (c < total) item_ptrs<SP, DP>(a, c, s, d);
    const unsigned long long sp = reinterpret_cast<unsigned long long>(s);
    const unsigned long long dp = reinterpret_cast<unsigned long long>(d);
    const int cnt = total - g < 32 ? int(total - g) : 32;
    for (int t = 0; t < cnt; ++t) {
      const char* st = reinterpret_cast<const char*>(__shfl_sync(0xffffffffu, sp, t));
      char* dt = reinterpret_cast<char*>(__shfl_sync(0xffffffffu, dp, t));
      for (uint32_t v0 = 0; v0 < vecs; v0 += 32 * kWarpUnroll) {
        uint4 x[kWarpUnroll];
#pragma unroll
        for (int u = 0; u < kWarpUnroll; ++u) {
          const uint32_t v = v0 + u * 32 + lane;
          if (v < vecs) x[u] = ld_stream(st + uint64_t(v) * 16);
        }
#pragma unroll
        for (int u = 0; u < kWarpUnroll; ++u) {
          const uint32_t v = v0 + u * 32 + lane;
          if (v < vecs) st_stream(dt + uint64_t(v) * 16, x[u]);
        }
      }
    }
  }
}

// ------------------------------------------------------------------------------------ BULK
constexpr int kBulkStages = 6;
constexpr uint32_t kBulkPiece = 32768;
constexpr int kBulkSmem = kBulkStages * kBulkPiece;  // 192 KiB -> one CTA per SM

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void bulk_load(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

__device__ __forceinline__ void bulk_store(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(ssrc)),
               "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

#ifdef AEG_BW_EVICT_FIRST  // experiment: streaming L2 policy on the BULKW bulk copies
__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ void bulk_load_ef(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar,
                                             uint64_t pol) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void bulk_store_ef(void* gdst, const void* ssrc, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(gdst),
               "r"(smem_u32(ssrc)), "r"(bytes), "l"(pol)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
#endif

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

template <bool SP, bool DP>
__global__ void __launch_bounds__(32) copy_bulk(const CopyArgs a) {
  extern __shared__ __align__(128) char smem[];
  __shared__ __align__(8) uint64_t bar[kBulkStages];
  if (threadIdx.x != 0) return;
  const uint64_t ppc = (a.chunk + kBulkPiece - 1) / kBulkPiece;
  const uint64_t items = uint64_t(a.nl) * uint64_t(a.n) * ppc;
  if (blockIdx.x >= items) return;
  const uint64_t mine = (items - blockIdx.x + gridDim.x - 1) / gridDim.x;
  for (int i = 0; i < kBulkStages; ++i) mbar_init(&bar[i], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");

  auto piece = [&](uint64_t k, const char*& s, char*& d, uint32_t& bytes) {
    const uint64_t w = blockIdx.x + k * gridDim.x;
    const uint64_t c = w / ppc;
    const uint64_t off = (w - c * ppc) * kBulkPiece;
    item_ptrs<SP, DP>(a, c, s, d);
    s += off;
    d += off;
    const uint64_t rem = a.chunk - off;
    bytes = rem < kBulkPiece ? uint32_t(rem) : kBulkPiece;
  };
  const char* s;
  char* d;
  uint32_t nb;
  for (uint64_t k = 0; k < mine && k < uint64_t(kBulkStages); ++k) {
    piece(k, s, d, nb);
    bulk_load(smem + k * kBulkPiece, s, nb, &bar[k]);
  }
  for (uint64_t k = 0; k < mine; ++k) {
    const int st = int(k % kBulkStages);
    mbar_wait(&bar[st], uint32_t((k / kBulkStages) & 1));
    piece(k, s, d, nb);
    bulk_store(d, smem + uint64_t(st) * kBulkPiece, nb);
    if (k >= 1 && k - 1 + kBulkStages < mine) {
      bulk_wait_read<1>();  // the store of item k-1 has finished reading its stage
      const uint64_t kn = k - 1 + kBulkStages;
      const int sn = int((k - 1) % kBulkStages);
      piece(kn, s, d, nb);
      bulk_load(smem + uint64_t(sn) * kBulkPiece, s, nb, &bar[sn]);
    }
  }
  bulk_wait_all();
}

// ----------------------------------------------------------------------------------- BULKW
// Small chunks (<= 16 KiB) through the bulk-copy engine: the single-thread BULK above is issue-bound
// there (one table load, two 64-bit divisions and two cp.async.bulk per 8 KiB, serialised in one
// thread).  Here a CTA is kBwWarps independent warps, each with its own ring of whole-chunk stages
// in shared memory (kBwSmem / kBwWarps bytes).  A warp resolves the pointers of 32 of its items at
// once, one per lane (one coalesced block-table load), and lane 0 issues the bulk copies with the
// pointers broadcast by __shfl_sync; the ring refill is the BULK pipeline (mbarrier complete_tx for
// loads, bulk_group read-completion before a stage is reloaded).
// Geometry (tools/small_chunk_probe.cu sweeps, profiles/r02/bulkw_geometry_sweep.txt): 6 warps x
// 16 KiB of stages in a 96 KiB CTA, one CTA per SM (grid = 148), i.e. 2 stages of 8 KiB pieces per
// warp and ~96 KiB in flight per SM: 6.3-6.5 TB/s for 8 KiB-320 KiB chunks over 30 GB-spread tables,
// vs 5.9-6.1 with 192 KiB (4 warps x 48 KiB) or with two CTAs per SM — more bytes or more, smaller
// bulk copies in flight per SM lose DRAM efficiency on scattered blocks.
#ifndef AEG_BW_WARPS  // overridable by tools/small_chunk_probe.cu
#define AEG_BW_WARPS 6
#endif
#ifndef AEG_BW_SMEM_KIB
#define AEG_BW_SMEM_KIB 96
#endif
constexpr int kBwWarps = AEG_BW_WARPS;
#ifndef AEG_BW_MAX_STAGES
#define AEG_BW_MAX_STAGES 16
#endif
constexpr int kBwMaxStages = AEG_BW_MAX_STAGES;
constexpr int kBwSmem = AEG_BW_SMEM_KIB * 1024;

template <bool SP, bool DP>
__global__ void __launch_bounds__(kBwWarps * 32) copy_bulkw(const CopyArgs a, uint32_t piece) {
  extern __shared__ __align__(128) char smem[];
  __shared__ __align__(8) uint64_t bar[kBwWarps][kBwMaxStages];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t per_warp = uint32_t(kBwSmem / kBwWarps);
  const uint32_t stages = min(uint32_t(kBwMaxStages), per_warp / piece);
  char* ring = smem + uint64_t(warp) * per_warp;
  uint64_t* wb = bar[warp];
  const uint64_t ppc = (a.chunk + piece - 1) / piece;
  const uint64_t items = uint64_t(a.nl) * uint64_t(a.n) * ppc;
  const uint64_t W = uint64_t(gridDim.x) * kBwWarps;
  const uint64_t gw = uint64_t(blockIdx.x) * kBwWarps + warp;
  if (gw >= items) return;  // warp-uniform
  const uint64_t mine = (items - gw + W - 1) / W;
  if (lane == 0) {
    for (uint32_t i = 0; i < stages; ++i) mbar_init(&wb[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  // lane j of a batch holds the pointers of the warp's item 32 * batch + j
  auto resolve = [&](uint64_t j, const char*& s, char*& d, uint32_t& nb) {
    const uint64_t w = gw + j * W;
    const uint64_t c = w / ppc;
    const uint64_t off = (w - c * ppc) * piece;
    item_ptrs<SP, DP>(a, c, s, d);
    s += off;
    d += off;
    const uint64_t rem = a.chunk - off;
    nb = rem < piece ? uint32_t(rem) : piece;
  };
#ifdef AEG_BW_EVICT_FIRST
  const uint64_t pol = evict_first_policy();
#endif
  const char* ls = nullptr;
  char* sd = nullptr;
  uint32_t lnb = 0, snb = 0;
  uint64_t lbatch = ~0ull, sbatch = ~0ull;
  auto load = [&](uint64_t j, uint32_t st) {
    if ((j >> 5) != lbatch) {  // warp-uniform: j is the same in every lane
      lbatch = j >> 5;
      const uint64_t jj = (lbatch << 5) + lane;
      char* dd;
      if (jj < mine) resolve(jj, ls, dd, lnb);
    }
    const char* s = reinterpret_cast<const char*>(
        __shfl_sync(0xffffffffu, reinterpret_cast<unsigned long long>(ls), int(j & 31)));
    const uint32_t nb = __shfl_sync(0xffffffffu, lnb, int(j & 31));
#ifdef AEG_BW_EVICT_FIRST
    if (lane == 0) bulk_load_ef(ring + uint64_t(st) * piece, s, nb, &wb[st], pol);
#else
    if (lane == 0) bulk_load(ring + uint64_t(st) * piece, s, nb, &wb[st]);
#endif
  };
  auto store = [&](uint64_t j, uint32_t st) {
    if ((j >> 5) != sbatch) {
      sbatch = j >> 5;
      const uint64_t jj = (sbatch << 5) + lane;
      const char* ss;
      if (jj < mine) resolve(jj, ss, sd, snb);
    }
    char* d = reinterpret_cast<char*>(__shfl_sync(0xffffffffu, reinterpret_cast<unsigned long long>(sd), int(j & 31)));
    const uint32_t nb = __shfl_sync(0xffffffffu, snb, int(j & 31));
#ifdef AEG_BW_EVICT_FIRST
    if (lane == 0) bulk_store_ef(d, ring + uint64_t(st) * piece, nb, pol);
#else
    if (lane == 0) bulk_store(d, ring + uint64_t(st) * piece, nb);
#endif
  };
  for (uint64_t j = 0; j < mine && j < stages; ++j) load(j, uint32_t(j));
  uint32_t st = 0, phase = 0, prev = stages - 1;
  for (uint64_t k = 0; k < mine; ++k) {
    if (lane == 0) mbar_wait(&wb[st], phase);
    __syncwarp();
    store(k, st);
    if (k >= 1 && k - 1 + stages < mine) {
      if (lane == 0) bulk_wait_read<1>();  // the store of item k-1 has finished reading its stage
      load(k - 1 + stages, prev);
    }
    prev = st;
    if (++st == stages) {
      st = 0;
      phase ^= 1;
    }
  }
  if (lane == 0) bulk_wait_all();
}

template <bool SP, bool DP>
cudaError_t launch_t(const CopyArgs& a, int impl, int max_ctas, cudaStream_t s) {
  const uint64_t items_lsu = uint64_t(a.nl) * a.n * ((a.chunk + kLsuPiece - 1) / kLsuPiece);
  if (items_lsu == 0) return cudaSuccess;
  if (impl == IMPL_WARP) {
    const uint64_t groups = (uint64_t(a.nl) * a.n + 31) / 32;  // one warp per 32 chunks
    uint64_t grid = max_ctas > 0 ? uint64_t(max_ctas) : uint64_t(kSMs) * 8;
    const uint64_t need = (groups * 32 + kWarpThreads - 1) / kWarpThreads;
    if (grid > need) grid = need;
    copy_warp<SP, DP><<<unsigned(grid), kWarpThreads, 0, s>>>(a);
  } else if (impl == IMPL_BULKW) {
    static std::atomic<uint64_t> attr_set_w{0};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const uint64_t bit = 1ull << (dev & 63);
    if (!(attr_set_w.load() & bit)) {
      e = cudaFuncSetAttribute(copy_bulkw<SP, DP>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBwSmem);
      if (e != cudaSuccess) return e;
      attr_set_w.fetch_or(bit);
    }
    // whole chunks up to 8 KiB per stage (half a warp's share), larger chunks in 8 KiB pieces; at
    // least 2 stages per warp (the refill of a stage is issued one item after its store, so one
    // stage would never refill).  One CTA per SM: grid = 148 (the 96 KiB CTA would fit twice).
    const uint32_t cap = std::min<uint32_t>(16u << 10, uint32_t(kBwSmem / kBwWarps / 2) & ~15u);
    const uint32_t piece = a.chunk <= cap ? uint32_t(a.chunk) : cap;
    const uint64_t items = uint64_t(a.nl) * a.n * ((a.chunk + piece - 1) / piece);
#ifndef AEG_BW_GRID
#define AEG_BW_GRID kSMs
#endif
    uint64_t grid = max_ctas > 0 ? uint64_t(max_ctas) : uint64_t(AEG_BW_GRID);
    const uint64_t need = (items + kBwWarps - 1) / kBwWarps;  // one item per warp at least
    if (grid > need) grid = need;
    copy_bulkw<SP, DP><<<unsigned(grid), kBwWarps * 32, kBwSmem, s>>>(a, piece);
  } else if (impl == IMPL_BULK) {
    static std::atomic<uint64_t> attr_set{0};  // per-device bit: opt-in smem attribute applied
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const uint64_t bit = 1ull << (dev & 63);
    if (!(attr_set.load() & bit)) {
      e = cudaFuncSetAttribute(copy_bulk<SP, DP>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
      if (e != cudaSuccess) return e;
      attr_set.fetch_or(bit);
    }
    const uint64_t items = uint64_t(a.nl) * a.n * ((a.chunk + kBulkPiece - 1) / kBulkPiece);
    uint64_t grid = max_ctas > 0 ? uint64_t(max_ctas) : uint64_t(kSMs);
    if (grid > items) grid = items;
    copy_bulk<SP, DP><<<unsigned(grid), 32, kBulkSmem, s>>>(a);
  } else {
    uint64_t grid = max_ctas > 0 ? uint64_t(max_ctas) : uint64_t(kSMs) * 4;
    if (grid > items_lsu) grid = items_lsu;
    copy_lsu<SP, DP><<<unsigned(grid), kLsuThreads, 0, s>>>(a);
  }
  return cudaGetLastError();
}

// Block-table fetch: the transfer's table is read by the GPU straight from the pinned host mirror
// (zero-copy, ld.global.cv: never a stale cached line of host memory the CPU has rewritten) into
// the device table arena, on the kernel stream that then uses it.  Not a cudaMemcpyAsync: a copy
// engine serves H2D copies FIFO across streams, so a table upload queued behind a swap-in's
// gigabytes of H2D held the next swap-out's first gather until they drained.
__global__ void __launch_bounds__(256) fetch_table(uint2* __restrict__ dst, const uint2* src, uint64_t words) {
  for (uint64_t w = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; w < words; w += uint64_t(gridDim.x) * blockDim.x) {
    uint2 v;
    asm volatile("ld.global.cv.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(src + w));
    dst[w] = v;
  }
}

template <bool SP, bool DP>
cudaError_t preload_t() {
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, copy_lsu<SP, DP>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, copy_warp<SP, DP>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, copy_bulk<SP, DP>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, copy_bulkw<SP, DP>);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(copy_bulk<SP, DP>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(copy_bulkw<SP, DP>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBwSmem);
  return e;
}

}  // namespace

// Load every copy kernel into the current device's context now.  With CUDA's lazy module loading a
// kernel's first launch loads its module and waits for the device; on the hot path that is both a
// latency spike and a deadlock hazard when another kernel spin-waits (found by the gate tests).
cudaError_t launch_fetch_table(void* dst, const void* src_host, uint64_t bytes, cudaStream_t s) {
  const uint64_t words = bytes / 8;
  if (words == 0) return cudaSuccess;
  const uint64_t ctas = std::min<uint64_t>(64, (words + 255) / 256);
  fetch_table<<<unsigned(ctas), 256, 0, s>>>(static_cast<uint2*>(dst), static_cast<const uint2*>(src_host), words);
  return cudaGetLastError();
}

cudaError_t preload_kernels() {
  cudaFuncAttributes fa0;
  cudaError_t e0 = cudaFuncGetAttributes(&fa0, fetch_table);
  if (e0 != cudaSuccess) return e0;
  cudaError_t e = preload_t<true, false>();
  if (e == cudaSuccess) e = preload_t<false, true>();
  if (e == cudaSuccess) e = preload_t<true, true>();
  if (e == cudaSuccess) e = preload_t<false, false>();
  return e;
}

cudaError_t launch_copy(const CopyArgs& a, int impl, int max_ctas, cudaStream_t s) {
  const bool sp = a.src_off != nullptr, dp = a.dst_off != nullptr;
  if (sp && dp) return launch_t<true, true>(a, impl, max_ctas, s);
  if (sp) return launch_t<true, false>(a, impl, max_ctas, s);
  if (dp) return launch_t<false, true>(a, impl, max_ctas, s);
  return launch_t<false, false>(a, impl, max_ctas, s);
}

// memmove semantics (reading 21): when the ranges overlap, copy in chunks of at most |dst - src|
// bytes, ascending when dst < src and descending when dst > src, each chunk one launch on the
// same stream so a chunk never reads bytes an earlier chunk overwrote.
cudaError_t launch_memmove(char* base, uint64_t src_off, uint64_t dst_off, uint64_t bytes, int impl,
                           cudaStream_t s, int* launches) {
  *launches = 0;
  if (bytes == 0 || src_off == dst_off) return cudaSuccess;
  const uint64_t gap = src_off > dst_off ? src_off - dst_off : dst_off - src_off;
  const uint64_t step = gap >= bytes ? bytes : gap;
  const uint64_t nchunks = (bytes + step - 1) / step;
  for (uint64_t q = 0; q < nchunks; ++q) {
    const uint64_t k = dst_off < src_off ? q : nchunks - 1 - q;
    const uint64_t off = k * step;
    const uint64_t len = (bytes - off) < step ? (bytes - off) : step;
    CopyArgs a;
    a.src = base + src_off + off;
    a.dst = base + dst_off + off;
    a.chunk = len;
    a.nl = 1;
    a.n = 1;
    cudaError_t e = launch_copy(a, impl, 0, s);
    if (e != cudaSuccess) return e;
    ++*launches;
  }
  return cudaSuccess;
}

}  // namespace aeg
