// extern "C" entry points of libaegkv.so (include/aeg.h).  Each one converts internal exceptions
// into an AEG_ERR_* code and a thread-local message; nothing throws across the ABI.
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <string>

#include "runtime/engine.h"

using aeg::Ctx;
using aeg::Error;

struct aeg_ctx_s {
  Ctx c;
};

namespace {

thread_local std::string g_err;

template <class F>
int guarded(F&& f) {
  try {
    g_err.clear();
    return f();
  } catch (const Error& e) {
    g_err = e.what();
    return e.code;
  } catch (const std::bad_alloc&) {
    g_err = "host out of memory";
    return AEG_ERR_OOM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return AEG_ERR_STATE;
  }
}

Ctx& C(aeg_ctx x) {
  AEG_REQUIRE(x, AEG_ERR_INVALID, "context is NULL");
  return x->c;
}

void set_device(Ctx& c) {
  if (!c.host_only) CUDA_TRY(cudaSetDevice(c.device));
}

// Run one data-path enqueue; if it throws after its transfer was created, drain and mark it failed
// (Ctx::abort_enqueue) so no reader can block on an event that will never be recorded.
template <class F>
uint64_t enqueue(Ctx& c, F&& f) {
  c.enqueuing = nullptr;
  try {
    const uint64_t x = f();
    c.enqueuing = nullptr;
    return x;
  } catch (...) {
    c.abort_enqueue();
    throw;
  }
}

constexpr uint32_t kIpcMagic = 0xAE6A1BC1u, kXferMagic = 0xAE6A1BC2u;

struct IpcBlob {
  uint32_t magic, version;
  int32_t pid, device;
  uint64_t raw_base;  // dev_kv in the exporter's address space
  uint64_t pool_bytes, slab_bytes;
  int32_t layout, pad;
  cudaIpcMemHandle_t mem;
  // shared CPU KV region (AEG_CFG_SHARED_HOST), empty name if none
  char shm[64];
  uint64_t host_bytes, host_slab_bytes, host_kv_bytes;
  int32_t host_layout, pad2;
};

struct XferBlobHead {
  uint32_t magic;
  int32_t pid;
  int32_t L;
  int32_t ipc;
  uint64_t id;
  // swap-out D2H pieces (Xfer::pev), exported so a peer's swap-in waits per piece too: after the
  // L + 1 layer/done handles come (npiece + 1) int32 piece starts, L * npiece event handles and the
  // n written host handles in transfer order (0 pieces: nothing follows).
  int32_t npiece;
  int32_t n;
  uint64_t serial;  // exporter's process-wide transfer serial (same-process imports pin it)
};

uint64_t xfer_blob_bytes(int32_t L, int32_t npiece, int32_t n) {
  uint64_t b = sizeof(XferBlobHead) + uint64_t(L + 1) * sizeof(cudaIpcEventHandle_t);
  if (npiece > 1)
    b += uint64_t(npiece + 1) * 4 + uint64_t(L) * uint64_t(npiece) * sizeof(cudaIpcEventHandle_t) + uint64_t(n) * 8;
  return b;
}

}  // namespace

extern "C" {

const char* aeg_last_error(void) { return g_err.c_str(); }

int aeg_config_default(aeg_config* cfg) {
  return guarded([&] {
    AEG_REQUIRE(cfg, AEG_ERR_INVALID, "cfg is NULL");
    std::memset(cfg, 0, sizeof *cfg);
    cfg->dev_slab_bytes = 1ull << 30;
    cfg->host_slab_bytes = 1ull << 30;
    cfg->stage_ring_bytes = 2ull << 30;  // "Stage Buffer (2 GB)"
    cfg->stage_chunk_bytes = 64ull << 20;
    cfg->staging_slot_bytes = 1ull << 30;  // one launch per layer for 7B-class batches (profiles/r01)
    cfg->staging_slots = 3;
    cfg->table_arena_bytes = 64ull << 20;
    cfg->host_threads = 8;
    cfg->dev_slab_layout = AEG_LAYER_MAJOR;
    cfg->host_slab_layout = AEG_LAYER_MAJOR;
    cfg->kernel = AEG_KERNEL_AUTO;
    cfg->dma_piece_mib = 128;
    cfg->pack_layer_mib = 32;  // per-request swaps of small layers (bench per_request_sync)
    return AEG_OK;
  });
}

int aeg_init(int device, const aeg_config* cfg, aeg_ctx* out) {
  return guarded([&] {
    AEG_REQUIRE(cfg && out, AEG_ERR_INVALID, "NULL argument");
    aeg_config c = *cfg;
    aeg_config d;
    aeg_config_default(&d);
    if (!c.dev_slab_bytes) c.dev_slab_bytes = d.dev_slab_bytes;
    if (!c.host_slab_bytes) c.host_slab_bytes = d.host_slab_bytes;
    if (!c.stage_ring_bytes) c.stage_ring_bytes = d.stage_ring_bytes;
    if (!c.stage_chunk_bytes) c.stage_chunk_bytes = d.stage_chunk_bytes;
    if (!c.staging_slot_bytes) c.staging_slot_bytes = d.staging_slot_bytes;
    if (!c.staging_slots) c.staging_slots = d.staging_slots;
    if (!c.table_arena_bytes) c.table_arena_bytes = d.table_arena_bytes;
    if (!c.host_threads) c.host_threads = d.host_threads;
    if (!c.dma_piece_mib) c.dma_piece_mib = d.dma_piece_mib;
    if (!c.pack_layer_mib) c.pack_layer_mib = d.pack_layer_mib;
    auto* x = new aeg_ctx_s();
    try {
      x->c.init(device, c);
    } catch (...) {
      try {
        x->c.shutdown();
      } catch (...) {
      }
      delete x;
      throw;
    }
    *out = x;
    return AEG_OK;
  });
}

int aeg_shutdown(aeg_ctx ctx) {
  return guarded([&] {
    if (!ctx) return AEG_OK;
    ctx->c.shutdown();
    delete ctx;
    return AEG_OK;
  });
}

int aeg_kv_alloc(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, int32_t n, aeg_block* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    c.poll();  // on-demand step ⑧ (reading 9)
    c.pool[pool].reclaim();
    c.pool[pool].alloc(sh, n, out);
    return AEG_OK;
  });
}

int aeg_kv_free(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    c.poll();
    c.pool[pool].free(blocks, n);
    return AEG_OK;
  });
}

int aeg_reclaim(aeg_ctx ctx, int blocking) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::unique_lock<std::mutex> g(c.mu);
    set_device(c);
    if (blocking && !c.host_only) {
      c.cv.wait(g, [&] { return c.w_inflight == 0; });
      for (auto& kv : c.xfers)
        if (kv.second->done_recorded && !kv.second->complete.load()) CUDA_TRY(cudaEventSynchronize(kv.second->done_ev));
    }
    c.housekeeping();
    return AEG_OK;
  });
}

int aeg_stats(aeg_ctx ctx, int32_t pool, aeg_pool_stats* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    c.pool[pool].stats(out);
    return AEG_OK;
  });
}

int aeg_block_info(aeg_ctx ctx, aeg_block b, int32_t* pool, uint32_t* slab, uint32_t* index) {
  return guarded([&] {
    (void)C(ctx);
    if (pool) *pool = aeg::block_pool(b);
    if (slab) *slab = aeg::block_slab(b);
    if (index) *index = aeg::block_idx(b);
    return AEG_OK;
  });
}

int aeg_block_ptr(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, aeg_block b, int32_t layer, void** p) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    AEG_REQUIRE(p, AEG_ERR_INVALID, "p is NULL");
    AEG_REQUIRE(!c.host_only, AEG_ERR_STATE, "host-only context has no memory");
    const aeg::Shape sh = aeg::Shape::from(shape);
    AEG_REQUIRE(layer >= 0 && layer < sh.L, AEG_ERR_INVALID, "layer out of range");
    std::lock_guard<std::mutex> g(c.mu);
    c.pool[pool].check_owned(&b, 1, &sh);
    char* base = pool == AEG_POOL_DEVICE ? c.dev_kv : c.host_kv;
    *p = base + c.pool[pool].off0(b, sh) + uint64_t(layer) * c.pool[pool].lstride(sh);
    return AEG_OK;
  });
}

int aeg_block_offsets(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, const aeg_block* blocks, int32_t n,
                      uint64_t* off0, uint64_t* layer_stride) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    AEG_REQUIRE((n == 0 || off0) && layer_stride, AEG_ERR_INVALID, "NULL output");
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    c.pool[pool].check_owned(blocks, n, &sh, false);
    for (int32_t i = 0; i < n; ++i) off0[i] = c.pool[pool].off0(blocks[i], sh);
    *layer_stride = c.pool[pool].lstride(sh);
    return AEG_OK;
  });
}

int aeg_pool_region(aeg_ctx ctx, int32_t pool, void** base, uint64_t* bytes) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    if (base) *base = pool == AEG_POOL_DEVICE ? c.dev_kv : c.host_kv;
    if (bytes) *bytes = c.pool[pool].pool_bytes;
    return AEG_OK;
  });
}

int aeg_peer_region(aeg_ctx ctx, int32_t peer, void** base, uint64_t* bytes) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    auto it = c.peers.find(peer);
    AEG_REQUIRE(it != c.peers.end() && it->second->valid, AEG_ERR_INVALID, "peer %d not imported", peer);
    if (base) *base = it->second->dev_kv;
    if (bytes) *bytes = it->second->geom.pool_bytes;
    return AEG_OK;
  });
}

int aeg_kv_swap_out(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* dev, const aeg_block* host, int32_t n,
                    uint32_t flags, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    *out = enqueue(c, [&] { return c.swap_out(sh, dev, host, n, flags); });
    return AEG_OK;
  });
}

int aeg_kv_swap_in(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* host, const aeg_block* dev, int32_t n,
                   uint32_t flags, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    *out = enqueue(c, [&] { return c.swap_in(sh, host, dev, n, flags); });
    return AEG_OK;
  });
}

int aeg_kv_migrate(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* src, int32_t peer, const aeg_block* dst,
                   int32_t n, uint32_t flags, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    *out = enqueue(c, [&] { return c.migrate(sh, src, peer, dst, n, flags); });
    return AEG_OK;
  });
}

int aeg_kv_swap_in_from(aeg_ctx ctx, const aeg_kv_shape* shape, int32_t peer, const aeg_block* peer_host,
                        const aeg_block* dev, int32_t n, aeg_xfer after, uint32_t flags, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    const aeg::Shape sh = aeg::Shape::from(shape);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    *out = enqueue(c, [&] { return c.swap_in_from(sh, peer, peer_host, dev, n, after, flags); });
    return AEG_OK;
  });
}

int aeg_kv_free_after(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n, aeg_xfer after) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    c.poll();
    c.pool[pool].free_after(blocks, n, after);
    return AEG_OK;
  });
}

int aeg_stream_fence(aeg_ctx ctx, void* stream) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(!c.host_only, AEG_ERR_STATE, "host-only context");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    CUDA_TRY(cudaEventRecord(c.fence_ev, s));
    c.tr_record(s, c.fence_ev);
    for (cudaStream_t t : {c.s_gather, c.s_d2h, c.s_h2d, c.s_scatter, c.s_weights, c.s_migrate, c.s_p2p}) {
      CUDA_TRY(cudaStreamWaitEvent(t, c.fence_ev, 0));
      c.tr_wait(t, c.fence_ev);
    }
    return AEG_OK;
  });
}

int aeg_layer_ready(aeg_ctx ctx, aeg_xfer x, int32_t layer, int32_t mode, void* stream) {
  return guarded([&] {
    Ctx& c = C(ctx);
    set_device(c);
    return c.layer_ready(x, layer, mode, static_cast<cudaStream_t>(stream));
  });
}

int aeg_xfer_layers(aeg_ctx ctx, aeg_xfer x, int32_t* layers) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(layers, AEG_ERR_INVALID, "layers is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    *layers = c.get_xfer(x)->L;
    return AEG_OK;
  });
}

int aeg_xfer_release(aeg_ctx ctx, aeg_xfer x) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    c.get_xfer(x)->released = true;
    return AEG_OK;
  });
}

int aeg_weights_stage(aeg_ctx ctx, const aeg_weight_desc* descs, int32_t n, int32_t tp_rank, int32_t tp_size,
                      uint64_t* dev_offsets_out, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    *out = c.weights_stage(descs, n, tp_rank, tp_size, dev_offsets_out);
    return AEG_OK;
  });
}

int aeg_weights_reset(aeg_ctx ctx, uint64_t offset) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    AEG_REQUIRE(offset <= c.cfg.device_weight_bytes && offset % 256 == 0, AEG_ERR_INVALID, "bad bump offset");
    c.w_bump = offset;
    return AEG_OK;
  });
}

int aeg_weights_region(aeg_ctx ctx, void** base, uint64_t* bytes, uint64_t* bump) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    if (base) *base = c.dev_w;
    if (bytes) *bytes = c.cfg.device_weight_bytes;
    if (bump) *bump = c.w_bump;
    return AEG_OK;
  });
}

int aeg_weights_relocate(aeg_ctx ctx, uint64_t src_off, uint64_t dst_off, uint64_t bytes, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    std::unique_lock<std::mutex> g(c.mu);
    set_device(c);
    // rule ❷: the prefetched bytes must have been issued on s_weights before the move
    c.cv.wait(g, [&] { return c.w_inflight == 0; });
    *out = enqueue(c, [&] { return c.relocate(src_off, dst_off, bytes); });
    return AEG_OK;
  });
}

int aeg_weights_stats(aeg_ctx ctx, uint64_t* chunks, double* issuer_wait_fill_ms, double* fill_wait_slot_ms) {
  return guarded([&] {
    Ctx& c = C(ctx);
    c.weights_counters(chunks, issuer_wait_fill_ms, fill_wait_slot_ms);
    return AEG_OK;
  });
}

int aeg_host_register(aeg_ctx ctx, void* ptr, uint64_t bytes) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(!c.host_only, AEG_ERR_STATE, "host-only context");
    AEG_REQUIRE(ptr && bytes, AEG_ERR_INVALID, "bad range");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    CUDA_TRY(cudaHostRegister(ptr, bytes, cudaHostRegisterPortable));
    c.registered.emplace_back(static_cast<char*>(ptr), bytes);
    return AEG_OK;
  });
}

int aeg_host_unregister(aeg_ctx ctx, void* ptr) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::unique_lock<std::mutex> g(c.mu);
    set_device(c);
    c.cv.wait(g, [&] { return c.w_inflight == 0; });
    CUDA_TRY(cudaStreamSynchronize(c.s_weights));
    for (size_t i = 0; i < c.registered.size(); ++i)
      if (c.registered[i].first == ptr) {
        CUDA_TRY(cudaHostUnregister(ptr));
        c.registered.erase(c.registered.begin() + long(i));
        return AEG_OK;
      }
    aeg::fail(AEG_ERR_INVALID, "range not registered");
  });
}

// --------------------------------------------------------------------------------- IPC / peers
int aeg_export_ipc(aeg_ctx ctx, void* buf, uint64_t* len) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(len, AEG_ERR_INVALID, "len is NULL");
    AEG_REQUIRE(!c.host_only, AEG_ERR_STATE, "host-only context");
    if (!buf) {
      *len = sizeof(IpcBlob);
      return AEG_OK;
    }
    AEG_REQUIRE(*len >= sizeof(IpcBlob), AEG_ERR_INVALID, "buffer too small");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    IpcBlob b{};
    b.magic = kIpcMagic;
    b.version = AEG_ABI_VERSION;
    b.pid = int32_t(getpid());
    b.device = c.device;
    b.raw_base = reinterpret_cast<uint64_t>(c.dev_kv);
    b.pool_bytes = c.pool[AEG_POOL_DEVICE].pool_bytes;
    b.slab_bytes = c.pool[AEG_POOL_DEVICE].slab_bytes;
    b.layout = c.pool[AEG_POOL_DEVICE].layout;
    CUDA_TRY(cudaIpcGetMemHandle(&b.mem, c.dev_mem));
    if (!c.shm_name.empty()) {
      std::snprintf(b.shm, sizeof b.shm, "%s", c.shm_name.c_str());
      b.host_bytes = c.host_kv_mapped;
      b.host_kv_bytes = c.pool[AEG_POOL_HOST].pool_bytes;
      b.host_slab_bytes = c.pool[AEG_POOL_HOST].slab_bytes;
      b.host_layout = c.pool[AEG_POOL_HOST].layout;
    }
    std::memcpy(buf, &b, sizeof b);
    *len = sizeof b;
    return AEG_OK;
  });
}

int aeg_import_peer(aeg_ctx ctx, int32_t peer, const void* buf, uint64_t len) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(peer >= 0 && peer < 64, AEG_ERR_INVALID, "peer index out of range");
    AEG_REQUIRE(buf && len >= sizeof(IpcBlob), AEG_ERR_INVALID, "bad blob");
    AEG_REQUIRE(!c.host_only, AEG_ERR_STATE, "host-only context");
    IpcBlob b;
    std::memcpy(&b, buf, sizeof b);
    AEG_REQUIRE(b.magic == kIpcMagic && b.version == AEG_ABI_VERSION, AEG_ERR_INVALID, "not an aegkv IPC blob");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    auto p = std::make_unique<aeg::Peer>();
    p->device = b.device;
    p->same_process = b.pid == int32_t(getpid());
    p->geom.init(AEG_POOL_DEVICE, b.pool_bytes, b.slab_bytes, b.layout);
    if (p->same_process) {
      p->dev_kv = reinterpret_cast<char*>(b.raw_base);
      if (b.device != c.device) {
        int can = 0;
        CUDA_TRY(cudaDeviceCanAccessPeer(&can, c.device, b.device));
        AEG_REQUIRE(can, AEG_ERR_CUDA, "device %d cannot access peer device %d", c.device, b.device);
        cudaError_t e = cudaDeviceEnablePeerAccess(b.device, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled)
          (void)cudaGetLastError();
        else
          CUDA_TRY(e);
      }
    } else {
      void* ptr = nullptr;
      CUDA_TRY(cudaIpcOpenMemHandle(&ptr, b.mem, cudaIpcMemLazyEnablePeerAccess));
      p->ipc_base = static_cast<char*>(ptr);
      p->dev_kv = p->ipc_base;  // dev_kv is the start of the exporter's allocation
    }
    if (b.shm[0] && !p->same_process) {  // the peer's part of the node-shared CPU KV cache
      b.shm[sizeof b.shm - 1] = 0;
      p->host_kv = aeg::map_shared_host(b.shm, b.host_bytes, false);
      p->host_bytes = b.host_bytes;
      p->host_geom.init(AEG_POOL_HOST, b.host_kv_bytes, b.host_slab_bytes, b.host_layout);
      p->has_host = true;
    }
    p->valid = true;
    auto it = c.peers.find(peer);
    if (it != c.peers.end()) {
      if (it->second->ipc_base) cudaIpcCloseMemHandle(it->second->ipc_base);
      if (it->second->has_host) aeg::unmap_shared_host(it->second->host_kv, it->second->host_bytes);
      p->events = std::move(it->second->events);
    }
    c.peers[peer] = std::move(p);
    return AEG_OK;
  });
}

int aeg_xfer_export(aeg_ctx ctx, aeg_xfer xid, void* buf, uint64_t* len) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(len, AEG_ERR_INVALID, "len is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    aeg::Xfer* x = c.get_xfer(xid);
    AEG_REQUIRE(x->done_recorded, AEG_ERR_STATE, "transfer not fully enqueued yet");
    const int32_t np = x->npiece > 1 ? x->npiece : 0;
    const int32_t nb = np ? int32_t(x->wpos.size()) : 0;
    const uint64_t need = xfer_blob_bytes(x->L, np, nb);
    if (!buf) {
      *len = need;
      return AEG_OK;
    }
    AEG_REQUIRE(*len >= need, AEG_ERR_INVALID, "buffer too small");
    set_device(c);
    AEG_REQUIRE(!x->released, AEG_ERR_STATE, "transfer already released");
    XferBlobHead h{kXferMagic, int32_t(getpid()), x->L, x->ipc ? 1 : 0, x->id, np, nb,
                   x->serial};
    char* o = static_cast<char*>(buf);
    std::memcpy(o, &h, sizeof h);
    auto put_event = [&](cudaIpcEventHandle_t* hd, cudaEvent_t e) {
      if (x->ipc) {
        CUDA_TRY(cudaIpcGetEventHandle(hd, e));
      } else {
        std::memset(hd, 0, sizeof *hd);
        std::memcpy(hd, &e, sizeof e);  // same-process peers use the event directly
      }
    };
    cudaIpcEventHandle_t* hs = reinterpret_cast<cudaIpcEventHandle_t*>(o + sizeof h);
    for (int32_t l = 0; l <= x->L; ++l) put_event(&hs[l], l < x->L ? x->ev[l] : x->done_ev);
    if (np) {
      char* q = o + sizeof h + uint64_t(x->L + 1) * sizeof(cudaIpcEventHandle_t);
      std::memcpy(q, x->piece_lo.data(), uint64_t(np + 1) * 4);
      q += uint64_t(np + 1) * 4;
      cudaIpcEventHandle_t* ps = reinterpret_cast<cudaIpcEventHandle_t*>(q);
      for (size_t k = 0; k < x->pev.size(); ++k) put_event(&ps[k], x->pev[k]);
      q += x->pev.size() * sizeof(cudaIpcEventHandle_t);
      std::vector<aeg_block> hb(size_t(nb), 0);
      for (auto& kv : x->wpos) hb[size_t(kv.second)] = kv.first;
      std::memcpy(q, hb.data(), uint64_t(nb) * 8);
    }
    *len = need;
    return AEG_OK;
  });
}

int aeg_xfer_import(aeg_ctx ctx, int32_t peer, const void* buf, uint64_t len, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(out && buf && len >= sizeof(XferBlobHead), AEG_ERR_INVALID, "bad arguments");
    XferBlobHead h;
    std::memcpy(&h, buf, sizeof h);
    AEG_REQUIRE(h.magic == kXferMagic, AEG_ERR_INVALID, "not an aegkv transfer blob");
    // bounds first (a shape has at most 4096 layers, a piece at least one block), so the size
    // arithmetic below cannot overflow on a malformed blob
    AEG_REQUIRE(h.L >= 0 && h.L <= 4096 && h.n >= 0 && h.npiece >= 0 && h.npiece <= std::max(h.n, 1),
                AEG_ERR_INVALID, "malformed transfer blob");
    AEG_REQUIRE(len >= xfer_blob_bytes(h.L, h.npiece, h.n), AEG_ERR_INVALID, "blob truncated");
    const bool same = h.pid == int32_t(getpid());
    AEG_REQUIRE(same || h.ipc, AEG_ERR_INVALID, "transfer events are not interprocess-capable");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    AEG_REQUIRE(peer >= 0 && peer < 64, AEG_ERR_INVALID, "peer index out of range");
    auto it = c.peers.find(peer);
    if (it == c.peers.end())  // events only: the importer need not map the exporter's pool
      it = c.peers.emplace(peer, std::make_unique<aeg::Peer>()).first;
    aeg::Peer* P = it->second.get();
    const cudaIpcEventHandle_t* hs =
        reinterpret_cast<const cudaIpcEventHandle_t*>(static_cast<const char*>(buf) + sizeof h);
    auto x = std::make_unique<aeg::Xfer>();
    x->id = c.next_xid++;
    x->serial = aeg::xfer_next_serial();
    x->kind = aeg::X_IMPORTED;
    x->L = h.L;
    x->owns_events = false;
    x->recorded.assign(h.L, 1);
    x->ev.resize(h.L);
    auto get_event = [&](const cudaIpcEventHandle_t& hd) {
      cudaEvent_t e;
      if (same) {
        std::memcpy(&e, &hd, sizeof e);
      } else {
        std::string key(reinterpret_cast<const char*>(&hd), sizeof hd);
        auto f = P->events.find(key);
        if (f == P->events.end()) {
          CUDA_TRY(cudaIpcOpenEventHandle(&e, hd));
          P->events.emplace(key, e);
        } else {
          e = f->second;
        }
      }
      return e;
    };
    for (int32_t l = 0; l <= h.L; ++l) {
      cudaEvent_t e = get_event(hs[l]);
      if (l < h.L)
        x->ev[l] = e;
      else
        x->done_ev = e;
    }
    if (h.npiece > 1) {
      const char* q = static_cast<const char*>(buf) + sizeof h + uint64_t(h.L + 1) * sizeof(cudaIpcEventHandle_t);
      x->piece_lo.resize(size_t(h.npiece) + 1);
      std::memcpy(x->piece_lo.data(), q, uint64_t(h.npiece + 1) * 4);
      q += uint64_t(h.npiece + 1) * 4;
      AEG_REQUIRE(x->piece_lo.front() == 0 && x->piece_lo.back() == h.n &&
                      std::is_sorted(x->piece_lo.begin(), x->piece_lo.end()),
                  AEG_ERR_INVALID, "bad piece table in transfer blob");
      const cudaIpcEventHandle_t* ps = reinterpret_cast<const cudaIpcEventHandle_t*>(q);
      x->pev.resize(size_t(h.L) * size_t(h.npiece));
      for (size_t k = 0; k < x->pev.size(); ++k) x->pev[k] = get_event(ps[k]);
      q += x->pev.size() * sizeof(cudaIpcEventHandle_t);
      std::vector<aeg_block> hb(size_t(h.n));
      std::memcpy(hb.data(), q, uint64_t(h.n) * 8);
      x->wpos.reserve(hb.size() * 2);
      for (int32_t i = 0; i < h.n; ++i) x->wpos.emplace(hb[size_t(i)], i);
      x->npiece = h.npiece;
    }
    x->done_recorded = true;
    if (same) {  // keep the exporter's events alive until this import is reaped
      x->pinned_serial = h.serial;
      aeg::xfer_pin_add(h.serial);
    }
    *out = x->id;
    c.xfers.emplace(x->id, std::move(x));
    return AEG_OK;
  });
}

// ------------------------------------------------------------------------------ instrumentation
int aeg_kernel_stats(aeg_ctx ctx, int32_t kind, uint64_t* launches, uint64_t* bytes, double* ms) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(kind >= 0 && kind < 5, AEG_ERR_INVALID, "bad kernel kind");
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    c.resolve_timing(true);
    if (launches) *launches = c.kstats[kind].launches;
    if (bytes) *bytes = c.kstats[kind].bytes;
    if (ms) *ms = c.kstats[kind].ms;
    return AEG_OK;
  });
}

int aeg_set_migrate_ctas(aeg_ctx ctx, int32_t ctas) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(ctas >= 0, AEG_ERR_INVALID, "ctas must be >= 0");
    std::lock_guard<std::mutex> g(c.mu);
    c.cfg.migrate_ctas = ctas;
    return AEG_OK;
  });
}

int aeg_kernel_stats_reset(aeg_ctx ctx) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    set_device(c);
    c.resolve_timing(true);
    for (auto& k : c.kstats) k = aeg::KStat{};
    return AEG_OK;
  });
}

int aeg_trace_enable(aeg_ctx ctx, int on) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    c.tracing = on != 0;
    return AEG_OK;
  });
}

int aeg_trace_read(aeg_ctx ctx, char* buf, uint64_t* len) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(len, AEG_ERR_INVALID, "len is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    if (!buf || *len < c.trace.size() + 1) {
      *len = c.trace.size() + 1;
      aeg::fail(AEG_ERR_INVALID, "buffer too small: need %llu bytes", (unsigned long long)(c.trace.size() + 1));
    }
    std::memcpy(buf, c.trace.c_str(), c.trace.size() + 1);
    *len = c.trace.size();
    c.trace.clear();
    return AEG_OK;
  });
}

int aeg_debug_xfer_begin(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n, aeg_xfer* out) {
  return guarded([&] {
    Ctx& c = C(ctx);
    AEG_REQUIRE(c.host_only, AEG_ERR_STATE, "debug transfers need a host-only context");
    AEG_REQUIRE(pool == AEG_POOL_DEVICE || pool == AEG_POOL_HOST, AEG_ERR_INVALID, "bad pool %d", pool);
    AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
    std::lock_guard<std::mutex> g(c.mu);
    c.pool[pool].check_owned(blocks, n, nullptr, false);
    aeg::Xfer* x = c.new_xfer(aeg::X_DEBUG, 1, false);
    for (int32_t i = 0; i < n; ++i) c.pool[pool].note_read(blocks[i], x->id);
    *out = x->id;
    return AEG_OK;
  });
}

int aeg_debug_xfer_complete(aeg_ctx ctx, aeg_xfer xid) {
  return guarded([&] {
    Ctx& c = C(ctx);
    std::lock_guard<std::mutex> g(c.mu);
    aeg::Xfer* x = c.get_xfer(xid);
    AEG_REQUIRE(x->kind == aeg::X_DEBUG, AEG_ERR_STATE, "not a debug transfer");
    x->debug_done = true;
    x->complete.store(true);
    return AEG_OK;
  });
}

}  // extern "C"
