// Block-table copy kernels for sm_100a (H2 gather, H4 scatter, H5 migrate, N1 relocate).
//
// One launch copies, for every layer t in [0, nl) and block i in [0, n), `chunk` bytes (Cl, one
// block's slice of one layer) from src to dst.  A side is "paged" when its table is given:
//   paged      addr = base + off[i] + (l_first + t) * lstride      (off[i] = layer-0 offset)
//   contiguous addr = base + (t * n + i) * chunk                    (layer-major staging image)
// Pure byte movement: 16-byte vectors, never through floating point (reading 14).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

namespace aeg {

struct CopyArgs {
  const char* src = nullptr;
  char* dst = nullptr;
  const uint64_t* src_off = nullptr;  // device array [n] or nullptr (contiguous)
  const uint64_t* dst_off = nullptr;
  uint64_t src_lstride = 0, dst_lstride = 0;
  uint64_t chunk = 0;                 // bytes per (block, layer); multiple of 16
  int32_t nl = 0, n = 0;
  int32_t l_first = 0;                // absolute layer of t = 0 (paged sides)
};

enum CopyImpl { IMPL_LSU = 1, IMPL_BULK = 2, IMPL_WARP = 3, IMPL_BULKW = 4 };

// Launch on `s`.  max_ctas <= 0: one full wave of the chosen kernel.  Returns the CUDA error of
// the launch.  `impl` is IMPL_LSU (registers, 16 B ld.global.nc / st.global) or IMPL_BULK
// (cp.async.bulk global->smem->global, mbarrier pipeline, one issuing thread per CTA).
cudaError_t launch_copy(const CopyArgs& a, int impl, int max_ctas, cudaStream_t s);

// Copy a block table (bytes, multiple of 8) from pinned, device-mapped host memory to device
// memory with a small kernel on `s` (zero-copy reads; no copy engine).
cudaError_t launch_fetch_table(void* dst, const void* src_host, uint64_t bytes, cudaStream_t s);

// Load all copy kernels (and set the BULK shared-memory attribute) for the current device.
cudaError_t preload_kernels();

// memmove inside one buffer (N1): overlap-safe ascending / descending chunking.
cudaError_t launch_memmove(char* base, uint64_t src_off, uint64_t dst_off, uint64_t bytes, int impl,
                           cudaStream_t s, int* launches);

}  // namespace aeg
