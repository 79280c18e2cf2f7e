// Context lifetime, transfers/events (rule ❶ readiness), the reclaim daemon (step ⑧), the block-
// table arena, kernel timing and the primitive trace.
#include "engine.h"

#include <fcntl.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <cctype>
#include <fstream>

#include <algorithm>
#include <chrono>
#include <cinttypes>
#include <cstring>

namespace aeg {

namespace {
constexpr uint64_t kMiB = 1ull << 20;
constexpr uint64_t kAlign = 2 * kMiB;

// Page-lock `bytes` of host memory once at init.  cudaHostAlloc faults and
// pins pages on one thread (~2.5 GB/s measured on the B200 box); instead: anonymous mmap with
// transparent huge pages, first touch from several threads, then cudaHostRegister of the populated
// range (~19 GB/s measured, same DMA bandwidth) — 41 GiB pin in ~2 s instead of ~17 s.
// Bind [p, p+bytes) to NUMA node `node` (>= 0) before first touch, so pages land next to the GPU's
// PCIe root (raw mbind syscall: no libnuma dependency).  Best effort: failure leaves first-touch.
void bind_numa(void* p, uint64_t bytes, int node) {
  if (node < 0 || node >= 1024) return;
  unsigned long mask[1024 / (8 * sizeof(unsigned long))] = {};
  mask[node / (8 * sizeof(unsigned long))] |= 1ul << (node % (8 * sizeof(unsigned long)));
  constexpr int kMpolBind = 2;
  syscall(SYS_mbind, p, bytes, kMpolBind, mask, 1024ul, 0u);
}

char* pin_host(uint64_t bytes, int node) {
  void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  AEG_REQUIRE(p != MAP_FAILED, AEG_ERR_OOM, "mmap of %llu host bytes failed", (unsigned long long)bytes);
  madvise(p, bytes, MADV_HUGEPAGE);
  bind_numa(p, bytes, node);
  char* b = static_cast<char*>(p);
  const unsigned T = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  std::vector<std::thread> th;
  for (unsigned i = 0; i < T; ++i)
    th.emplace_back([=] {
      for (uint64_t o = bytes * i / T / 4096 * 4096; o < bytes * (i + 1) / T; o += 4096) b[o] = 0;
    });
  for (auto& t : th) t.join();
  cudaError_t e = cudaHostRegister(b, bytes, cudaHostRegisterPortable | cudaHostRegisterMapped);
  if (e != cudaSuccess) {
    munmap(b, bytes);
    fail(AEG_ERR_CUDA, "cudaHostRegister of %llu bytes failed: %s", (unsigned long long)bytes, cudaGetErrorString(e));
  }
  void* dp = nullptr;
  CUDA_TRY(cudaHostGetDevicePointer(&dp, b, 0));
  AEG_REQUIRE(dp == b, AEG_ERR_CUDA, "registered host memory is not addressable at the same pointer on the device");
  return b;
}

void unpin_host(char* b, uint64_t bytes) {
  cudaHostUnregister(b);
  munmap(b, bytes);
}

void touch(char* b, uint64_t bytes) {
  const unsigned T = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  std::vector<std::thread> th;
  for (unsigned i = 0; i < T; ++i)
    th.emplace_back([=] {
      for (uint64_t o = bytes * i / T / 4096 * 4096; o < bytes * (i + 1) / T; o += 4096) b[o] = 0;
    });
  for (auto& t : th) t.join();
}

void register_same_ptr(char* b, uint64_t bytes) {
  CUDA_TRY(cudaHostRegister(b, bytes, cudaHostRegisterPortable | cudaHostRegisterMapped));
  void* dp = nullptr;
  CUDA_TRY(cudaHostGetDevicePointer(&dp, b, 0));
  AEG_REQUIRE(dp == b, AEG_ERR_CUDA, "registered host memory is not addressable at the same pointer on the device");
}
}  // namespace

// The node-shared Unified CPU KV Cache (Fig. 5; NEXT-2): a POSIX shared-memory object
// mapped by every instance of the node, page-locked once per process.
char* map_shared_host(const std::string& name, uint64_t bytes, bool create, int numa_node) {
  int fd = shm_open(name.c_str(), create ? (O_CREAT | O_EXCL | O_RDWR) : O_RDWR, 0600);
  AEG_REQUIRE(fd >= 0, AEG_ERR_INVALID, "shm_open(%s) failed", name.c_str());
  if (create && ftruncate(fd, off_t(bytes)) != 0) {
    close(fd);
    shm_unlink(name.c_str());
    fail(AEG_ERR_OOM, "ftruncate of shared host region %s failed", name.c_str());
  }
  void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  AEG_REQUIRE(p != MAP_FAILED, AEG_ERR_OOM, "mmap of shared host region %s failed", name.c_str());
  char* b = static_cast<char*>(p);
  if (create) {
    bind_numa(b, bytes, numa_node);
    touch(b, bytes);
  }
  try {
    register_same_ptr(b, bytes);
  } catch (...) {
    munmap(b, bytes);
    if (create) shm_unlink(name.c_str());
    throw;
  }
  return b;
}

void unmap_shared_host(char* b, uint64_t bytes) {
  cudaHostUnregister(b);
  munmap(b, bytes);
}

// ------------------------------------------------------------------------------------ init
constexpr double kVramReserveFrac = 0.10;  // left free for the caller's tensors

void Ctx::init(int dev, const aeg_config& c) {
  cfg = c;
  host_only = (cfg.flags & AEG_CFG_HOST_ONLY) != 0;
  timing = (cfg.flags & AEG_CFG_TIMING) != 0;
  AEG_REQUIRE(cfg.dev_slab_bytes > 0 && cfg.host_slab_bytes > 0, AEG_ERR_INVALID, "slab sizes must be > 0");
  if (!host_only && cfg.device_kv_bytes == 0) {
    // Reading 22: the self-managed buffer takes "all the necessary VRAM ... in
    // one allocation, leaving around 10% free memory for tensor libraries".  device_kv_bytes = 0
    // sizes the KV region so that the whole allocation (KV + weights + staging rings + tables) is
    // 90% of the device's free memory, rounded down to whole slabs.
    CUDA_TRY(cudaSetDevice(dev));
    CUDA_TRY(cudaFree(nullptr));
    size_t fr = 0, tot = 0;
    CUDA_TRY(cudaMemGetInfo(&fr, &tot));
    const uint64_t others = align_up(cfg.device_weight_bytes, kAlign) +
                            2 * align_up(cfg.staging_slot_bytes * uint64_t(cfg.staging_slots), kAlign) +
                            align_up(cfg.table_arena_bytes, kAlign);
    const uint64_t budget = uint64_t(double(fr) * (1.0 - kVramReserveFrac));
    AEG_REQUIRE(budget > others + cfg.dev_slab_bytes, AEG_ERR_OOM,
                "90%% of free VRAM (%llu bytes) does not hold the other regions plus one slab",
                (unsigned long long)budget);
    cfg.device_kv_bytes = (budget - others) / cfg.dev_slab_bytes * cfg.dev_slab_bytes;
  }
  pool[AEG_POOL_DEVICE].init(AEG_POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, cfg.dev_slab_layout);
  pool[AEG_POOL_HOST].init(AEG_POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, cfg.host_slab_layout);
  for (auto& p : pool) {
    p.is_done = [this](uint64_t x) { return is_done(x); };
    p.done_below = &done_below;
  }
  if (host_only) {
    if (!(cfg.flags & AEG_CFG_NO_DAEMON)) daemon = std::thread([this] { daemon_loop(); });
    return;
  }
  device = dev;
  CUDA_TRY(cudaSetDevice(device));
  CUDA_TRY(cudaFree(nullptr));  // create / retain the primary context
  CUDA_TRY(preload_kernels());   // no lazy module load on the data path
  AEG_REQUIRE(cfg.kernel >= AEG_KERNEL_AUTO && cfg.kernel <= AEG_KERNEL_BULKW, AEG_ERR_INVALID,
              "unknown kernel selection %d", cfg.kernel);
  AEG_REQUIRE(cfg.staging_slots >= 2, AEG_ERR_INVALID, "need at least 2 staging slots");
  AEG_REQUIRE(cfg.staging_slot_bytes >= 1 * kMiB && cfg.staging_slot_bytes % 256 == 0, AEG_ERR_INVALID,
              "staging slot must be >= 1 MiB and 256-byte aligned");
  AEG_REQUIRE(cfg.stage_chunk_bytes >= 1 * kMiB && cfg.stage_ring_bytes >= 2 * cfg.stage_chunk_bytes,
              AEG_ERR_INVALID, "stage ring must hold >= 2 chunks of >= 1 MiB");

  // One device allocation: [KV | weights | out ring | in ring | tables]
  const uint64_t kv = align_up(cfg.device_kv_bytes, kAlign);
  const uint64_t w = align_up(cfg.device_weight_bytes, kAlign);
  const uint64_t ring = align_up(cfg.staging_slot_bytes * cfg.staging_slots, kAlign);
  const uint64_t tab = align_up(cfg.table_arena_bytes, kAlign);
  dev_mem_bytes = kv + w + 2 * ring + tab;
  CUDA_TRY(cudaMalloc(&dev_mem, dev_mem_bytes));
  dev_kv = dev_mem;
  dev_w = dev_mem + kv;
  ring_out.base = dev_mem + kv + w;
  ring_in.base = ring_out.base + ring;
  tables.dev = ring_in.base + ring;
  tables.bytes = tab;

  // One pinned host allocation, pinned once: [CPU KV | Stage Buffer | tables]
  const uint64_t hkv = align_up(cfg.host_kv_bytes, kAlign);
  const uint64_t hst = align_up(cfg.stage_ring_bytes, kAlign);
  // NUMA placement of all pinned memory: next to the GPU's PCIe root unless told otherwise
  int numa = cfg.numa_node > 0 ? cfg.numa_node - 1 : -1;
  if (cfg.numa_node == 0) {
    char bus[64] = {0};
    if (cudaDeviceGetPCIBusId(bus, sizeof bus, device) == cudaSuccess) {
      for (char* q = bus; *q; ++q) *q = char(std::tolower(*q));
      std::ifstream f(std::string("/sys/bus/pci/devices/") + bus + "/numa_node");
      if (!(f >> numa)) numa = -1;
    }
  }
  numa_bound = numa;
  if (cfg.flags & AEG_CFG_SHARED_HOST) {
    static std::atomic<int> seq{0};
    shm_name = "/aegkv." + std::to_string(getpid()) + "." + std::to_string(seq++);
    host_kv = map_shared_host(shm_name, hkv, true, numa);
    host_kv_mapped = hkv;
    host_mem_bytes = hst + tab;
    host_mem = pin_host(host_mem_bytes, numa);
    host_stage = host_mem;
  } else {
    host_mem_bytes = hkv + hst + tab;
    host_mem = pin_host(host_mem_bytes, numa);
    host_kv = host_mem;
    host_stage = host_mem + hkv;
  }
  tables.host = host_stage + hst;

  int lo = 0, hi = 0;
  CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  // copy-engine streams and the kernel streams; the gather/scatter/migrate kernels get the highest
  // priority so they never queue behind long decode kernels of the caller.
  CUDA_TRY(cudaStreamCreateWithPriority(&s_gather, cudaStreamNonBlocking, hi));
  CUDA_TRY(cudaStreamCreateWithPriority(&s_scatter, cudaStreamNonBlocking, hi));
  CUDA_TRY(cudaStreamCreateWithPriority(&s_migrate, cudaStreamNonBlocking, hi));
  CUDA_TRY(cudaStreamCreateWithFlags(&s_d2h, cudaStreamNonBlocking));
  CUDA_TRY(cudaStreamCreateWithFlags(&s_h2d, cudaStreamNonBlocking));
  CUDA_TRY(cudaStreamCreateWithFlags(&s_weights, cudaStreamNonBlocking));
  CUDA_TRY(cudaStreamCreateWithFlags(&s_p2p, cudaStreamNonBlocking));
  CUDA_TRY(cudaEventCreateWithFlags(&fence_ev, cudaEventDisableTiming));
  for (Ring* r : {&ring_out, &ring_in}) {
    r->slot_bytes = cfg.staging_slot_bytes;
    r->bytes = cfg.staging_slot_bytes * uint64_t(cfg.staging_slots);
  }
  weights_start();
  if (!(cfg.flags & AEG_CFG_NO_DAEMON)) daemon = std::thread([this] { daemon_loop(); });
}

void Ctx::shutdown() {
  if (!host_only) {
    weights_stop();
    cudaSetDevice(device);
    for (cudaStream_t s : {s_gather, s_d2h, s_h2d, s_scatter, s_weights, s_migrate, s_p2p})
      if (s) cudaStreamSynchronize(s);
  }
  {
    std::lock_guard<std::mutex> g(mu);
    stop = true;
  }
  cv.notify_all();
  if (daemon.joinable()) daemon.join();
  if (host_only) return;
  for (auto& kv : xfers) {
    Xfer* x = kv.second.get();
    if (x->pinned_serial) xfer_pin_drop(x->pinned_serial);
    // still imported by a same-process context (aeg.h: exporters outlive imports): leak its
    // events rather than destroy events that context may still wait on
    if (!x->owns_events || xfer_pinned(x->serial)) continue;
    for (cudaEvent_t e : x->ev) cudaEventDestroy(e);
    if (x->done_ev) cudaEventDestroy(x->done_ev);
  }
  xfers.clear();
  for (cudaEvent_t e : ev_pool) cudaEventDestroy(e);
  for (cudaEvent_t e : ev_pool_ipc) cudaEventDestroy(e);
  for (cudaEvent_t e : timing_pool) cudaEventDestroy(e);
  for (auto& t : pending_timing) {
    cudaEventDestroy(t.a);
    cudaEventDestroy(t.b);
  }
  ring_out.destroy();
  ring_in.destroy();
  for (auto& kv : peers) {
    Peer* p = kv.second.get();
    for (auto& e : p->events) cudaEventDestroy(e.second);
    if (p->ipc_base) cudaIpcCloseMemHandle(p->ipc_base);
    if (p->has_host) unmap_shared_host(p->host_kv, p->host_bytes);
  }
  if (!shm_name.empty()) {
    unmap_shared_host(host_kv, host_kv_mapped);
    shm_unlink(shm_name.c_str());
  }
  for (auto& r : registered) cudaHostUnregister(r.first);
  cudaEventDestroy(fence_ev);
  for (cudaStream_t s : {s_gather, s_d2h, s_h2d, s_scatter, s_weights, s_migrate, s_p2p})
    if (s) cudaStreamDestroy(s);
  if (dev_mem) cudaFree(dev_mem);
  if (host_mem) unpin_host(host_mem, host_mem_bytes);
}

// --------------------------------------------------------------------------- staging ring
char* Ring::acquire(uint64_t size, cudaStream_t producer, cudaEvent_t* full, cudaEvent_t* freed, uint64_t* off,
                   std::vector<cudaEvent_t>* waited) {
  AEG_REQUIRE(size > 0 && size <= slot_bytes, AEG_ERR_INVALID, "staging segment of %llu bytes exceeds a slot",
              (unsigned long long)size);
  // segments start on 16 KiB boundaries (the trace's ring granule, swap.cc ring_cells): two
  // segments never share a granule, so ring reuse is exactly what the rule checker sees
  constexpr uint64_t kRingAlign = 16u << 10;
  head += (kRingAlign - (head % bytes) % kRingAlign) % kRingAlign;
  const uint64_t pos = head % bytes;
  if (pos + size > bytes) head += bytes - pos;  // never wrap inside a segment
  const uint64_t start = head, end = head + size;
  // every older segment that started before end - bytes shares bytes with [start, end)
  while (!live.empty() && end > bytes && live.front().start < end - bytes) {
    Seg& s = live.front();
    CUDA_TRY(cudaStreamWaitEvent(producer, s.freed, 0));
    if (waited) waited->push_back(s.freed);
    pool.push_back(s.full);   // both events were already waited on; safe to re-record
    pool.push_back(s.freed);
    live.pop_front();
  }
  auto take = [&]() {
    if (!pool.empty()) {
      cudaEvent_t e = pool.back();
      pool.pop_back();
      return e;
    }
    cudaEvent_t e;
    CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    return e;
  };
  Seg s{start, end, take(), take()};
  live.push_back(s);
  head = end;
  *full = s.full;
  *freed = s.freed;
  *off = start % bytes;
  return base + start % bytes;
}

void Ring::destroy() {
  for (auto& s : live) {
    cudaEventDestroy(s.full);
    cudaEventDestroy(s.freed);
  }
  for (cudaEvent_t e : pool) cudaEventDestroy(e);
  live.clear();
  pool.clear();
}

// ------------------------------------------------------------------------------- daemon ⑧
void Ctx::daemon_loop() {
  if (!host_only) cudaSetDevice(device);
  std::unique_lock<std::mutex> lk(mu);
  while (!stop) {
    housekeeping();
    cv.wait_for(lk, std::chrono::milliseconds(1));
  }
}

bool Ctx::is_done(uint64_t x) {
  auto it = xfers.find(x);
  return it == xfers.end() || it->second->complete.load(std::memory_order_acquire);
}

void Ctx::poll() {
  poll_events();
  uint64_t lo = next_xid;  // the lowest id still incomplete bounds the completed prefix
  for (auto& kv : xfers)
    if (!kv.second->complete.load(std::memory_order_acquire)) lo = std::min(lo, kv.first);
  done_below = lo;
}

void Ctx::poll_events() {
  if (host_only) {
    for (auto& kv : xfers)
      if (kv.second->debug_done) kv.second->complete.store(true);
    return;
  }
  for (auto& kv : xfers) {
    Xfer* x = kv.second.get();
    if (x->complete.load() || !x->done_recorded) continue;
    cudaError_t e = cudaEventQuery(x->done_ev);
    if (e == cudaSuccess) {
      x->complete.store(true, std::memory_order_release);
      if (tracing) {
        char b[64];
        snprintf(b, sizeof b, "sync %p", (void*)x->done_ev);
        tr(b);
      }
    } else if (e != cudaErrorNotReady) {
      (void)cudaGetLastError();
    }
  }
}

void Ctx::housekeeping() {
  poll();
  pool[0].reclaim();
  pool[1].reclaim();
  // release table-arena ranges of completed transfers (FIFO)
  while (!tables.live.empty() && is_done(tables.live.front().xid)) tables.live.pop_front();
  // reap released + completed transfers, recycle their events
  for (auto it = xfers.begin(); it != xfers.end();) {
    Xfer* x = it->second.get();
    if (x->released && x->complete.load() && !xfer_pinned(x->serial)) {
      if (x->pinned_serial) xfer_pin_drop(x->pinned_serial);
      if (x->owns_events && !host_only) {
        for (cudaEvent_t e : x->ev) give_event(e, x->ipc);
        if (x->done_ev) give_event(x->done_ev, x->ipc);
        for (cudaEvent_t e : x->pev) give_event(e, x->ipc);
      }
      it = xfers.erase(it);
    } else {
      ++it;
    }
  }
  if (++sweep % 64 == 0) {
    pool[0].forget_completed();
    pool[1].forget_completed();
  }
  cv.notify_all();
}

// -------------------------------------------------------------------------------- events
cudaEvent_t Ctx::take_event(bool ipc) {
  auto& p = ipc ? ev_pool_ipc : ev_pool;
  if (!p.empty()) {
    cudaEvent_t e = p.back();
    p.pop_back();
    return e;
  }
  cudaEvent_t e;
  CUDA_TRY(cudaEventCreateWithFlags(&e, ipc ? (cudaEventDisableTiming | cudaEventInterprocess) : cudaEventDisableTiming));
  return e;
}

void Ctx::give_event(cudaEvent_t e, bool ipc) { (ipc ? ev_pool_ipc : ev_pool).push_back(e); }

namespace {
std::mutex g_pin_mu;
std::unordered_map<uint64_t, int32_t> g_pins;
std::atomic<uint64_t> g_serial{1};
}  // namespace

uint64_t xfer_next_serial() { return g_serial.fetch_add(1); }
void xfer_pin_add(uint64_t serial) {
  std::lock_guard<std::mutex> g(g_pin_mu);
  ++g_pins[serial];
}
void xfer_pin_drop(uint64_t serial) {
  std::lock_guard<std::mutex> g(g_pin_mu);
  auto it = g_pins.find(serial);
  if (it != g_pins.end() && --it->second <= 0) g_pins.erase(it);
}
bool xfer_pinned(uint64_t serial) {
  std::lock_guard<std::mutex> g(g_pin_mu);
  return g_pins.count(serial) != 0;
}

Xfer* Ctx::new_xfer(int kind, int32_t L, bool ipc) {
  auto x = std::make_unique<Xfer>();
  x->id = next_xid++;
  x->serial = xfer_next_serial();
  x->kind = kind;
  x->L = L;
  x->ipc = ipc;
  x->recorded.assign(L, 0);
  if (!host_only) {
    x->ev.resize(L);
    for (int32_t l = 0; l < L; ++l) x->ev[l] = take_event(ipc);
    x->done_ev = take_event(ipc);
  }
  Xfer* raw = x.get();
  xfers.emplace(raw->id, std::move(x));
  enqueuing = raw;
  return raw;
}

// A CUDA error interrupted an enqueue: some of the transfer's work may be queued, some not, and
// some events never recorded.  Drain the library streams (error path only), then mark every layer
// recorded + the transfer complete and failed, so no waiter blocks and readiness reports the error.
void Ctx::abort_enqueue() {
  Xfer* x = enqueuing;
  enqueuing = nullptr;
  if (!x || host_only) return;
  for (cudaStream_t s : {s_gather, s_d2h, s_h2d, s_scatter, s_migrate, s_p2p}) cudaStreamSynchronize(s);
  (void)cudaGetLastError();
  std::fill(x->recorded.begin(), x->recorded.end(), uint8_t(1));
  x->done_recorded = true;
  x->failed = true;
  x->released = true;  // the caller never received its id: reap it
  x->complete.store(true);
  cv.notify_all();
}

Xfer* Ctx::get_xfer(uint64_t id) {
  auto it = xfers.find(id);
  AEG_REQUIRE(it != xfers.end() && !it->second->released, AEG_ERR_STATE, "unknown or released transfer %llu",
              (unsigned long long)id);
  return it->second.get();
}

void Ctx::record(Xfer* x, int32_t layer, cudaStream_t s) {
  cudaEvent_t e = layer < 0 ? x->done_ev : x->ev[layer];
  CUDA_TRY(cudaEventRecord(e, s));
  tr_record(s, e);
  if (layer < 0)
    x->done_recorded = true;
  else
    x->recorded[layer] = 1;
}

// Rule ❷/❸: make stream s wait for the per-layer events [la, lb) of the incomplete transfers in
// deps (per-layer granularity, reading 12; transfers without matching layers: their done event).
void Ctx::wait_deps(cudaStream_t s, const std::vector<uint64_t>& deps, int32_t la, int32_t lb) {
  for (uint64_t d : deps) {
    auto it = xfers.find(d);
    if (it == xfers.end() || it->second->complete.load()) continue;
    Xfer* x = it->second.get();
    for (int32_t l = la; l < lb; ++l) {
      cudaEvent_t e;
      if (x->kind != X_WEIGHTS && x->kind != X_RELOCATE && x->L > l && x->recorded[l])
        e = x->ev[l];
      else if (x->done_recorded)
        e = x->done_ev;
      else
        fail(AEG_ERR_STATE, "dependency transfer %llu has unrecorded events", (unsigned long long)d);
      CUDA_TRY(cudaStreamWaitEvent(s, e, 0));
      tr_wait(s, e);
    }
  }
}

// Rule ❶ (Table 2).
int Ctx::layer_ready(uint64_t id, int32_t layer, int mode, cudaStream_t s) {
  std::unique_lock<std::mutex> lk(mu);
  Xfer* x = get_xfer(id);
  AEG_REQUIRE(layer >= -1 && layer < x->L, AEG_ERR_INVALID, "layer %d out of range [-1, %d)", layer, x->L);
  AEG_REQUIRE(mode >= AEG_READY_QUERY && mode <= AEG_READY_BLOCK, AEG_ERR_INVALID, "bad mode %d", mode);
  if (host_only) {
    AEG_REQUIRE(mode == AEG_READY_QUERY, AEG_ERR_STATE, "host-only context: QUERY only");
    return x->complete.load() ? AEG_OK : AEG_NOT_READY;
  }
  AEG_REQUIRE(!x->failed, AEG_ERR_CUDA, "transfer %llu failed while being enqueued", (unsigned long long)id);
  auto recorded = [&] { return layer < 0 ? x->done_recorded : x->recorded[layer] != 0; };
  if (!recorded()) {
    if (mode == AEG_READY_QUERY) return AEG_NOT_READY;
    // weights pipeline: the event is recorded when its chunk is issued; wait for that on the host
    cv.wait(lk, [&] { return recorded() || stop; });
    AEG_REQUIRE(recorded(), AEG_ERR_STATE, "context shut down");
  }
  cudaEvent_t e = layer < 0 ? x->done_ev : x->ev[layer];
  if (mode == AEG_READY_QUERY) {
    if (x->complete.load()) return AEG_OK;
    cudaError_t r = cudaEventQuery(e);
    if (r == cudaSuccess) return AEG_OK;
    if (r == cudaErrorNotReady) return AEG_NOT_READY;
    fail(AEG_ERR_CUDA, "cudaEventQuery: %s", cudaGetErrorString(r));
  }
  if (mode == AEG_READY_WAIT_STREAM) {
    CUDA_TRY(cudaStreamWaitEvent(s, e, 0));
    tr_wait(s, e);
    return AEG_OK;
  }
  lk.unlock();  // BLOCK: the transfer stays alive until released by this caller
  CUDA_TRY(cudaEventSynchronize(e));
  lk.lock();
  if (tracing) {
    char b[64];
    snprintf(b, sizeof b, "sync %p", (void*)e);
    tr(b);
  }
  return AEG_OK;
}

// --------------------------------------------------------------------------- table arena
// FIFO ring: live entries are [oldest.start, head) circularly.  A request that does not fit
// waits for the oldest transfers to complete.
uint64_t Ctx::alloc_table(uint64_t bytes, uint64_t xid, char** host, char** dev) {
  bytes = align_up(bytes, 256);
  AEG_REQUIRE(bytes <= tables.bytes / 2, AEG_ERR_INVALID, "block table of %llu bytes exceeds the arena",
              (unsigned long long)bytes);
  for (;;) {
    bool ok = false;
    uint64_t start = 0;
    if (tables.live.empty()) {
      tables.head = 0;
      ok = true;
    } else {
      const uint64_t oldest = tables.live.front().start;
      if (tables.head > oldest) {
        if (tables.head + bytes <= tables.bytes) {
          start = tables.head;
          ok = true;
        } else if (bytes <= oldest) {
          start = 0;
          ok = true;
        }
      } else if (tables.head + bytes <= oldest) {
        start = tables.head;
        ok = true;
      }
    }
    if (ok) {
      if (tables.live.empty()) start = 0;
      tables.head = start + bytes;
      tables.live.push_back({xid, start, tables.head});
      *host = tables.host + start;
      *dev = tables.dev + start;
      return start;
    }
    uint64_t oldest = tables.live.front().xid;
    auto it = xfers.find(oldest);
    if (it != xfers.end() && it->second->done_recorded) CUDA_TRY(cudaEventSynchronize(it->second->done_ev));
    housekeeping();
  }
}

// ----------------------------------------------------------------------- kernels + timing
void Ctx::fetch_table(char* dev, const char* host, uint64_t bytes, cudaStream_t s) {
  cudaError_t e = launch_fetch_table(dev, host, bytes, s);
  AEG_REQUIRE(e == cudaSuccess, AEG_ERR_CUDA, "table fetch launch failed: %s", cudaGetErrorString(e));
  kstats[4].launches++;
  kstats[4].bytes += bytes;
}

void Ctx::launch(int kind, const CopyArgs& a, cudaStream_t s, int impl, int max_ctas) {
  cudaEvent_t ta = nullptr, tb = nullptr;
  if (timing) {
    auto take = [&]() {
      if (!timing_pool.empty()) {
        cudaEvent_t e = timing_pool.back();
        timing_pool.pop_back();
        return e;
      }
      cudaEvent_t e;
      CUDA_TRY(cudaEventCreate(&e));
      return e;
    };
    ta = take();
    tb = take();
    CUDA_TRY(cudaEventRecord(ta, s));
  }
  cudaError_t e = launch_copy(a, impl, max_ctas, s);
  AEG_REQUIRE(e == cudaSuccess, AEG_ERR_CUDA, "copy kernel launch failed: %s", cudaGetErrorString(e));
  kstats[kind].launches++;
  kstats[kind].bytes += 2 * a.chunk * uint64_t(a.nl) * uint64_t(a.n);
  if (ta) {
    CUDA_TRY(cudaEventRecord(tb, s));
    pending_timing.push_back({kind, ta, tb});
    if (pending_timing.size() > 4096) resolve_timing(true);
  }
}

void Ctx::resolve_timing(bool block) {
  std::vector<TimingRec> keep;
  for (auto& t : pending_timing) {
    if (block) cudaEventSynchronize(t.b);
    float ms = 0;
    cudaError_t e = cudaEventElapsedTime(&ms, t.a, t.b);
    if (e == cudaSuccess) {
      kstats[t.kind].ms += ms;
      timing_pool.push_back(t.a);
      timing_pool.push_back(t.b);
    } else {
      (void)cudaGetLastError();
      keep.push_back(t);
    }
  }
  pending_timing.swap(keep);
}

// ---------------------------------------------------------------------------------- trace
std::string Ctx::sname(cudaStream_t s) const {
  if (s == s_gather) return "gather";
  if (s == s_d2h) return "d2h";
  if (s == s_h2d) return "h2d";
  if (s == s_scatter) return "scatter";
  if (s == s_weights) return "weights";
  if (s == s_migrate) return "migrate";
  if (s == s_p2p) return "p2p";
  char b[32];
  snprintf(b, sizeof b, "u%p", (void*)s);
  return b;
}

void Ctx::tr_record(cudaStream_t s, cudaEvent_t e) {
  if (!tracing) return;
  char b[96];
  snprintf(b, sizeof b, "record %s %p", sname(s).c_str(), (void*)e);
  tr(b);
}

void Ctx::tr_wait(cudaStream_t s, cudaEvent_t e) {
  if (!tracing) return;
  char b[96];
  snprintf(b, sizeof b, "wait %s %p", sname(s).c_str(), (void*)e);
  tr(b);
}

std::string Ctx::cells(int tag, const SlabPool& p, const aeg_block* b, int32_t n, int32_t la, int32_t lb,
                       int32_t i0, int32_t i1) const {
  (void)p;
  (void)n;
  std::string out;
  char buf[64];
  const char* t = tag == 0 ? "D" : tag == 1 ? "H" : "P";
  for (int32_t l = la; l < lb; ++l)
    for (int32_t i = i0; i < i1; ++i) {
      snprintf(buf, sizeof buf, "%s%s:%u:%u:%d", out.empty() ? "" : ",", t, block_slab(b[i]), block_idx(b[i]), l);
      out += buf;
    }
  return out;
}

}  // namespace aeg
