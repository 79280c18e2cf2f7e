/* A plain-C client of libaegkv.so: the boundary used without Python or PyTorch (include/aeg.h only;
 * the GPU mode also uses the CUDA runtime for its own test pattern and checks).
 *
 *   c_client host   allocator only (AEG_CFG_HOST_ONLY, no CUDA call): alloc / free / move-list stats
 *   c_client gpu    a Qwen-7B-shaped swap round trip: fill device blocks, swap out to host blocks,
 *                   swap back into fresh device blocks with per-layer readiness, compare every byte
 *
 * Build: gcc -O2 -I include -o c_client examples/c_client.c -L <lib dir> -laegkv -lcudart \
 *            -Wl,-rpath,<lib dir>                       (tests/test_c_client.py does this)
 * Exit status 0 on success; on failure the library's aeg_last_error() is printed. */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "aeg.h"

#define CHECK(call)                                                                          \
  do {                                                                                     \
    int rc_ = (call);                                                                      \
    if (rc_ < 0) {                                                                         \
      fprintf(stderr, "%s:%d: %s -> %d (%s)\n", __FILE__, __LINE__, #call, rc_, aeg_last_error()); \
      return 1;                                                                            \
    }                                                                                      \
  } while (0)

/* CUDA runtime entry points used by the GPU mode (declared here: no CUDA headers needed). */
int cudaMemcpy(void* dst, const void* src, size_t n, int kind);
int cudaDeviceSynchronize(void);

static int host_mode(void) {
  aeg_config cfg;
  CHECK(aeg_config_default(&cfg));
  cfg.flags = AEG_CFG_HOST_ONLY | AEG_CFG_NO_DAEMON;
  cfg.device_kv_bytes = 8ull << 20;
  cfg.host_kv_bytes = 8ull << 20;
  cfg.dev_slab_bytes = 1ull << 20;
  cfg.host_slab_bytes = 1ull << 20;
  aeg_ctx ctx;
  CHECK(aeg_init(0, &cfg, &ctx));
  aeg_kv_shape sh = {2, 4, 64, 2, 16}; /* configs[0]: 32 KiB blocks, 32 per 1 MiB slab */
  aeg_block a[40], b[8];
  CHECK(aeg_kv_alloc(ctx, AEG_POOL_DEVICE, &sh, 40, a));
  CHECK(aeg_kv_alloc(ctx, AEG_POOL_DEVICE, &sh, 8, b));
  aeg_pool_stats st;
  CHECK(aeg_stats(ctx, AEG_POOL_DEVICE, &st));
  if (st.owned_blocks != 48 || st.n_slabs - st.free_slabs != 2) {
    fprintf(stderr, "unexpected stats: owned %llu, assigned slabs %llu\n", (unsigned long long)st.owned_blocks,
            (unsigned long long)(st.n_slabs - st.free_slabs));
    return 1;
  }
  CHECK(aeg_kv_free(ctx, AEG_POOL_DEVICE, a, 40));
  if (aeg_kv_free(ctx, AEG_POOL_DEVICE, a, 1) >= 0) { /* double free must be refused */
    fprintf(stderr, "double free accepted\n");
    return 1;
  }
  CHECK(aeg_kv_free(ctx, AEG_POOL_DEVICE, b, 8));
  CHECK(aeg_stats(ctx, AEG_POOL_DEVICE, &st));
  if (st.owned_blocks != 0 || st.free_slabs != st.n_slabs || st.peak_assigned_bytes != 2ull << 20) {
    fprintf(stderr, "pool not empty after frees\n");
    return 1;
  }
  CHECK(aeg_shutdown(ctx));
  printf("c_client host: allocator OK\n");
  return 0;
}

static int gpu_mode(void) {
  aeg_config cfg;
  CHECK(aeg_config_default(&cfg));
  cfg.device_kv_bytes = 2ull << 30;
  cfg.host_kv_bytes = 1ull << 30;
  aeg_ctx ctx;
  CHECK(aeg_init(0, &cfg, &ctx));
  aeg_kv_shape sh = {32, 32, 128, 2, 16}; /* Qwen-7B: 256 KiB chunks, 8 MiB blocks */
  enum { N = 64, L = 32 };
  const uint64_t chunk = 256ull << 10;
  aeg_block dev[N], host[N], back[N];
  CHECK(aeg_kv_alloc(ctx, AEG_POOL_DEVICE, &sh, N, dev));
  CHECK(aeg_kv_alloc(ctx, AEG_POOL_HOST, &sh, N, host));
  CHECK(aeg_kv_alloc(ctx, AEG_POOL_DEVICE, &sh, N, back));
  void* dbase;
  uint64_t dbytes;
  CHECK(aeg_pool_region(ctx, AEG_POOL_DEVICE, &dbase, &dbytes));
  uint64_t off0[N], lstride;
  /* fill every (block, layer) chunk of `dev` with a pattern naming it */
  CHECK(aeg_block_offsets(ctx, AEG_POOL_DEVICE, &sh, dev, N, off0, &lstride));
  uint64_t* buf = (uint64_t*)malloc(chunk);
  for (int i = 0; i < N; ++i)
    for (int l = 0; l < L; ++l) {
      for (uint64_t w = 0; w < chunk / 8; ++w) buf[w] = ((uint64_t)i << 48) ^ ((uint64_t)l << 40) ^ w;
      if (cudaMemcpy((char*)dbase + off0[i] + l * lstride, buf, chunk, 4 /* default */) != 0) return 1;
    }
  aeg_xfer x, y;
  CHECK(aeg_kv_swap_out(ctx, &sh, dev, host, N, AEG_FREE_SRC, &x));
  CHECK(aeg_kv_swap_in(ctx, &sh, host, back, N, AEG_FREE_SRC, &y));
  for (int l = 0; l < L; ++l) CHECK(aeg_layer_ready(ctx, y, l, AEG_READY_BLOCK, NULL));
  CHECK(aeg_layer_ready(ctx, x, -1, AEG_READY_BLOCK, NULL));
  CHECK(aeg_block_offsets(ctx, AEG_POOL_DEVICE, &sh, back, N, off0, &lstride));
  uint64_t bad = 0;
  for (int i = 0; i < N; ++i)
    for (int l = 0; l < L; ++l) {
      if (cudaMemcpy(buf, (char*)dbase + off0[i] + l * lstride, chunk, 4) != 0) return 1;
      for (uint64_t w = 0; w < chunk / 8; ++w) bad += buf[w] != (((uint64_t)i << 48) ^ ((uint64_t)l << 40) ^ w);
    }
  free(buf);
  CHECK(aeg_xfer_release(ctx, x));
  CHECK(aeg_xfer_release(ctx, y));
  CHECK(aeg_shutdown(ctx));
  if (bad) {
    fprintf(stderr, "%llu words differ after the round trip\n", (unsigned long long)bad);
    return 1;
  }
  printf("c_client gpu: %d blocks x %d layers swapped out and back, every byte identical\n", N, L);
  return 0;
}

int main(int argc, char** argv) {
  if (argc > 1 && strcmp(argv[1], "gpu") == 0) return gpu_mode();
  return host_mode();
}
