// The per-(process, device) context behind aeg_ctx: pools, streams, staging rings, transfers,
// events, the reclaim daemon and the weight pipeline.  See DESIGN.md §2 for the data layout.
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <condition_variable>
#include <deque>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "../kernels/copy.h"
#include "common.h"
#include "slab.h"

namespace aeg {

#define CUDA_TRY(call)                                                                        \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess) ::aeg::fail(AEG_ERR_CUDA, "%s failed: %s", #call, cudaGetErrorString(e_)); \
  } while (0)

enum XferKind { X_SWAP_OUT = 0, X_SWAP_IN, X_MIGRATE, X_WEIGHTS, X_RELOCATE, X_DEBUG, X_IMPORTED };

// Shared (node-wide) CPU KV region: create (exporter) or map (importer), page-locked (engine.cc).
char* map_shared_host(const std::string& name, uint64_t bytes, bool create, int numa_node = -1);
void unmap_shared_host(char* b, uint64_t bytes);

// One transfer: one CUDA event per readiness layer (reading 11) + one completion event.
struct Xfer {
  uint64_t id = 0;
  int kind = 0;
  int32_t L = 0;
  bool ipc = false;                 // events are interprocess-capable
  std::vector<cudaEvent_t> ev;      // per layer
  std::vector<uint8_t> recorded;    // per layer: event recorded (monotone), guarded by ctx.mu
  cudaEvent_t done_ev = nullptr;
  bool done_recorded = false;
  std::atomic<bool> complete{false};
  bool released = false;
  bool owns_events = true;          // imported transfers borrow cached peer events
  // Same-process imports borrow the exporter's raw events: while a process-wide pin on `serial`
  // is held (xfer_pin_*) the exporter keeps this transfer and its events; an imported copy holds
  // the pin on `pinned_serial` until it is reaped or its context shuts down.
  uint64_t serial = 0;
  uint64_t pinned_serial = 0;
  bool failed = false;              // enqueue was interrupted by an error (events force-recorded)
  bool debug_done = false;          // host-only synthetic transfers
  uint64_t table_mark = 0;          // table-arena end offset to release on completion
  // Swap-out only: its D2H of each layer is issued as `npiece` block-range pieces; piece p covers
  // the transfer's blocks [piece_lo[p], piece_lo[p+1]) and pev[l * npiece + p] is recorded on the
  // D2H stream right after piece p of layer l (stream order: pieces of a layer land in index
  // order).  A swap-in reading those host blocks waits for the piece that wrote them instead of
  // the whole layer (rule ❷ at sub-layer granularity), so a round trip's H2D of layer l starts
  // one piece, not one layer, after the D2H of layer l began.
  int32_t npiece = 0;
  std::vector<int32_t> piece_lo;
  std::vector<cudaEvent_t> pev;
  std::unordered_map<aeg_block, int32_t> wpos;  // written host block -> its index in the transfer
};

// Process-wide pins of exported transfers (serial numbers), for same-process imports.
uint64_t xfer_next_serial();
void xfer_pin_add(uint64_t serial);
void xfer_pin_drop(uint64_t serial);
bool xfer_pinned(uint64_t serial);

// Device staging ring for one direction of KV swaps: a byte ring (slots x slot_bytes) in which
// segments of any size <= slot_bytes are packed back to back.  Reuse is ordered entirely on the
// GPU (rule ❸ at ring level, no host blocking): a new segment's producer stream waits on the
// `freed` events of the older segments whose bytes it overwrites; its consumer waits on `full`.
// Packing matters because one copy engine serves all H2D streams FIFO (profiles/r01/ce_probe.txt):
// a transfer of many small segments must be enqueued at once, not trickle in as fixed slots free up.
struct Ring {
  struct Seg {
    uint64_t start, end;  // monotonic byte positions
    cudaEvent_t full, freed;
  };
  char* base = nullptr;
  uint64_t slot_bytes = 0;  // max segment size
  uint64_t bytes = 0;       // ring size
  uint64_t head = 0;        // monotonic
  std::deque<Seg> live;
  std::vector<cudaEvent_t> pool;
  // Reserve `size` bytes; makes `producer` wait for the segments being overwritten.  Returns the
  // device pointer and the segment's (full, freed) events.
  char* acquire(uint64_t size, cudaStream_t producer, cudaEvent_t* full, cudaEvent_t* freed, uint64_t* off,
                std::vector<cudaEvent_t>* waited);
  void destroy();
};

// Device block-table arena (+ pinned host mirror), allocated FIFO per transfer and released when
// the transfer completes.
struct TableArena {
  char* dev = nullptr;
  char* host = nullptr;
  uint64_t bytes = 0, head = 0;
  struct Entry {
    uint64_t xid, start, end;
  };
  std::deque<Entry> live;  // FIFO order
};

struct Peer {
  bool valid = false;
  bool same_process = false;
  int device = -1;
  char* dev_kv = nullptr;          // mapped base of the peer's device KV region
  char* ipc_base = nullptr;        // what cudaIpcOpenMemHandle returned (to close)
  SlabPool geom;                   // geometry only (no ownership state)
  std::unordered_map<std::string, cudaEvent_t> events;  // opened IPC events, by handle bytes
  // the peer's shared CPU KV region (AEG_CFG_SHARED_HOST), mapped + page-locked here
  char* host_kv = nullptr;
  uint64_t host_bytes = 0;
  SlabPool host_geom;
  bool has_host = false;
};

struct KStat {
  uint64_t launches = 0, bytes = 0;
  double ms = 0;
};

struct TimingRec {
  int kind;
  cudaEvent_t a, b;
};

struct WeightPipe;  // weights.cc

struct Ctx {
  int device = -1;
  aeg_config cfg{};
  bool host_only = false;
  std::mutex mu;
  std::condition_variable cv;  // signalled when events get recorded / transfers complete

  SlabPool pool[2];
  // memory: one device allocation, one pinned host allocation
  char* dev_mem = nullptr;
  uint64_t dev_mem_bytes = 0;
  char* dev_kv = nullptr;
  char* dev_w = nullptr;
  char* host_mem = nullptr;
  uint64_t host_mem_bytes = 0;
  char* host_kv = nullptr;
  char* host_stage = nullptr;
  std::string shm_name;   // AEG_CFG_SHARED_HOST: POSIX shm object holding the CPU KV region
  int numa_bound = -1;    // NUMA node the pinned host memory was bound to (-1: first touch)
  uint64_t host_kv_mapped = 0;
  uint64_t w_bump = 0;
  int w_inflight = 0;

  cudaStream_t s_gather = nullptr, s_d2h = nullptr, s_h2d = nullptr, s_scatter = nullptr;
  cudaStream_t s_weights = nullptr, s_migrate = nullptr;
  cudaStream_t s_p2p = nullptr;  // copy-engine hand-off route (AEG_MIGRATE_CE): staging -> peer pool
  cudaEvent_t fence_ev = nullptr;
  Ring ring_out, ring_in;
  TableArena tables;

  std::unordered_map<uint64_t, std::unique_ptr<Xfer>> xfers;
  uint64_t done_below = 1;  // every transfer id below this has completed (updated by poll, under mu)
  uint64_t next_xid = 1;
  std::vector<cudaEvent_t> ev_pool, ev_pool_ipc;

  std::thread daemon;
  bool stop = false;
  int sweep = 0;  // housekeeping rounds (access-map pruning cadence)
  std::unique_ptr<WeightPipe> wp;
  std::unordered_map<int, std::unique_ptr<Peer>> peers;
  std::vector<std::pair<char*, uint64_t>> registered;

  bool timing = false;
  KStat kstats[5];   // gather, scatter, migrate, relocate, table fetch
  std::vector<TimingRec> pending_timing;
  std::vector<cudaEvent_t> timing_pool;

  bool tracing = false;
  std::string trace;

  // ---- lifetime (engine.cc)
  Ctx();
  ~Ctx();  // defined in weights.cc, where WeightPipe is complete
  void init(int dev, const aeg_config& c);
  void shutdown();
  void daemon_loop();

  // ---- transfers (engine.cc)
  bool is_done(uint64_t x);        // completion observed (or transfer already reaped)
  void poll();                     // poll_events + advance done_below (caller holds mu)
  void poll_events();              // query the completion events of in-flight transfers
  void housekeeping();             // poll + reclaim + release tables + reap (caller holds mu)
  Xfer* new_xfer(int kind, int32_t L, bool ipc);
  Xfer* enqueuing = nullptr;       // transfer whose enqueue is in progress (error recovery)
  void abort_enqueue();            // error path: drain library streams, mark the transfer failed
  Xfer* get_xfer(uint64_t id);     // STATE if unknown/released
  cudaEvent_t take_event(bool ipc);
  void give_event(cudaEvent_t e, bool ipc);
  void record(Xfer* x, int32_t layer, cudaStream_t s);   // layer -1 = done_ev
  void wait_deps(cudaStream_t s, const std::vector<uint64_t>& deps, int32_t la, int32_t lb);
  int layer_ready(uint64_t x, int32_t layer, int mode, cudaStream_t s);
  uint64_t alloc_table(uint64_t bytes, uint64_t xid, char** host, char** dev);
  void fetch_table(char* dev, const char* host, uint64_t bytes, cudaStream_t s);  // table -> device, kernel

  // ---- kernels / timing
  void launch(int kind, const CopyArgs& a, cudaStream_t s, int impl, int max_ctas);
  void resolve_timing(bool block);

  // ---- trace (engine.cc)
  std::string sname(cudaStream_t s) const;
  void tr(const std::string& line) {
    if (tracing) {
      trace += line;
      trace += '\n';
    }
  }
  void tr_record(cudaStream_t s, cudaEvent_t e);
  void tr_wait(cudaStream_t s, cudaEvent_t e);
  std::string cells(int pool_tag, const SlabPool& p, const aeg_block* b, int32_t n, int32_t la, int32_t lb,
                    int32_t i0, int32_t i1) const;

  // ---- data paths (swap.cc, weights.cc)
  uint64_t swap_out(const Shape& sh, const aeg_block* dev, const aeg_block* host, int32_t n, uint32_t flags);
  uint64_t swap_in(const Shape& sh, const aeg_block* host, const aeg_block* dev, int32_t n, uint32_t flags);
  // swap-in from a (possibly peer) host region with an extra per-layer dependency `after` (NEXT-2)
  uint64_t swap_in_from(const Shape& sh, int32_t peer, const aeg_block* host, const aeg_block* dev, int32_t n,
                        uint64_t after, uint32_t flags);
  uint64_t migrate(const Shape& sh, const aeg_block* src, int32_t peer, const aeg_block* dst, int32_t n,
                   uint32_t flags);
  uint64_t relocate(uint64_t src_off, uint64_t dst_off, uint64_t bytes);
  uint64_t weights_stage(const aeg_weight_desc* d, int32_t n, int32_t r, int32_t tp, uint64_t* offs);
  void weights_start();
  void weights_stop();
  void weights_counters(uint64_t* chunks, double* wait_fill_ms, double* wait_slot_ms);
};

}  // namespace aeg
