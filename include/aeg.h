/*
 * aeg.h — C ABI of libaegkv.so, the B200-native data-movement hot path under Aegaeon's
 * token-level auto-scaling (Xiang et al., SOSP '25; PAPER.md = /root/reference/PAPER.md).
 *
 * What sits behind this boundary:
 *   - a unified, slab-allocated paged KV cache in VRAM and in pinned DRAM
 *   - move lists (quarantine) + a daemon that reclaims them
 *   - swap-out  P->C: gather kernel + copy-engine D2H on the KV-Out stream
 *   - swap-in   C->D: copy-engine H2D + scatter kernel on the KV-In stream
 *   - prefill->decode hand-off over NVLink (fused gather -> remote store)      north star; 1433-1459
 *   - per-(transfer, layer) CUDA events enforcing rules ❶❷❸
 *   - chunked, pipelined, TP-sharded weight staging into a bump buffer
 *
 * Conventions (apply to every function unless stated otherwise)
 *   Return value : AEG_OK (0) on success; AEG_NOT_READY (1) only from QUERY-mode readiness;
 *                  negative AEG_ERR_* on failure.  aeg_last_error() returns a thread-local
 *                  message for the last failure on the calling thread.  No function aborts the
 *                  process or throws across the ABI.
 *   Ownership    : the library owns pools, staging rings, streams, events and its threads.
 *                  The caller owns every array it passes; inputs are copied before return;
 *                  outputs are written only when AEG_OK is returned.
 *   Asynchrony   : data calls (swap_out / swap_in / migrate / weights_stage / relocate) return
 *                  after enqueueing work on library streams.  Completion of layer l of a
 *                  transfer is observed ONLY through aeg_layer_ready (rule ❶).
 *   Threads      : every call is thread-safe (one mutex per context, shared with the daemon).
 *   Process model: one process per GPU.  Peers exchange aeg_export_ipc blobs out of band
 *                  (e.g. torch.distributed all_gather_object) and call aeg_import_peer.
 *
 * Block handles (aeg_block) are opaque to callers but stable: bits [63:62] pool
 * (0 device, 1 host), [61:32] slab index, [31:0] block index inside the slab.
 */
#ifndef AEG_H_
#define AEG_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define AEG_ABI_VERSION 1

typedef struct aeg_ctx_s* aeg_ctx; /* one per (process, device); library-owned */
typedef uint64_t aeg_block;        /* see encoding above */
typedef uint64_t aeg_xfer;         /* transfer id, > 0; 0 = none */

/* ---- enums ------------------------------------------------------------------------------ */
enum { AEG_POOL_DEVICE = 0, AEG_POOL_HOST = 1 };
enum { AEG_LAYER_MAJOR = 0, AEG_BLOCK_MAJOR = 1 };
enum {
  AEG_OK = 0,
  AEG_NOT_READY = 1,
  AEG_ERR_INVALID = -1, /* bad argument, shape mismatch, handle of another pool/shape   */
  AEG_ERR_OOM = -2,     /* not enough free (non-quarantined) blocks / region exhausted  */
  AEG_ERR_CUDA = -3,    /* a CUDA runtime call failed (message has the CUDA error)      */
  AEG_ERR_STATE = -4    /* unowned / double-freed block, unknown transfer, wrong mode   */
};
/* aeg_layer_ready modes (Table 2) */
enum {
  AEG_READY_QUERY = 0,       /* cudaEventQuery: AEG_OK if done, AEG_NOT_READY otherwise     */
  AEG_READY_WAIT_STREAM = 1, /* cudaStreamWaitEvent(stream, ev[l]); returns immediately    */
  AEG_READY_BLOCK = 2        /* cudaEventSynchronize(ev[l])                                 */
};
/* transfer flags */
enum {
  AEG_FREE_SRC = 1u << 0,  /* free the source blocks once enqueued; they sit in the move list
                              until the transfer completes               */
  AEG_NO_DEPS = 1u << 1,   /* caller guarantees ordering: skip last-writer stream waits (❷❸) */
  AEG_IPC_EVENTS = 1u << 2, /* interprocess-capable events, so aeg_xfer_export works across
                              processes (implied for AEG_CFG_SHARED_HOST contexts, for
                              aeg_kv_swap_in_from a peer and for migrates to another process)  */
  AEG_MIGRATE_CE = 1u << 3  /* aeg_kv_migrate only: the copy-engine route instead of the fused
                              kernel — gather kernel into the out staging ring, then copy-engine
                              commands into the destination pool (zero SMs on the link)         */
};
/* weight split kinds (Megatron-style tensor parallelism, reading 18) */
enum { AEG_SPLIT_REPLICATED = 0, AEG_SPLIT_COL = 1, AEG_SPLIT_ROW = 2, AEG_SPLIT_VOCAB = 3 };
/* config flags */
enum {
  AEG_CFG_HOST_ONLY = 1u << 0, /* no CUDA at all: allocator / bookkeeping only (CPU tests)   */
  AEG_CFG_NO_DAEMON = 1u << 1, /* no reclaim thread: reclaim only via aeg_reclaim            */
  AEG_CFG_TIMING = 1u << 2,    /* time every gather/scatter/migrate launch with CUDA events  */
  AEG_CFG_SHARED_HOST = 1u << 3 /* CPU KV region in POSIX shared memory, mappable by peers:
                                   the node-shared "Unified CPU KV Cache" (Fig. 5) */
};
/* kernel selection for gather/scatter/migrate.  AEG_KERNEL_AUTO picks the measured best by chunk
 * size Cl (profiles/r02/): gather/scatter WARP if Cl <= 2 KiB, otherwise BULKW (bulk
 * copies issued by 6 warps per CTA, one CTA per SM); migrate (paged -> paged) WARP if Cl <= 4 KiB,
 * else BULKW within this process's pools on this GPU and LSU (16-byte stores) into another
 * process's or another GPU's pool.  LSU / BULK (one issuing thread per CTA) / WARP / BULKW can be
 * forced for every launch. */
enum { AEG_KERNEL_AUTO = 0, AEG_KERNEL_LSU = 1, AEG_KERNEL_BULK = 2, AEG_KERNEL_WARP = 3, AEG_KERNEL_BULKW = 4 };

/* ---- structs ---------------------------------------------------------------------------- */

/* Per-token KV cache shape (L, 2, H, D) at elem_bytes each (Table 1);
 * a block holds block_tokens tokens of all L layers.  Cl = block_tokens*2*H*D*elem_bytes must
 * be a multiple of 16 bytes.  Two shapes are the same shape iff all five fields are equal. */
typedef struct {
  int32_t num_layers, num_kv_heads, head_dim, elem_bytes, block_tokens;
} aeg_kv_shape;

/* Sizes are bytes.  Zero fields take the defaults of aeg_config_default(). */
typedef struct {
  uint64_t device_kv_bytes;     /* unified GPU KV cache region (slabs).  0 = the paper's sizing
                                   (reading 22): the one device allocation
                                   takes 90% of free VRAM, the KV region gets what the other
                                   regions leave, in whole slabs (aeg_pool_region reports it)   */
  uint64_t device_weight_bytes; /* self-managed weights region (bump allocated)               */
  uint64_t host_kv_bytes;       /* unified CPU KV cache, pinned once at init  */
  uint64_t dev_slab_bytes;      /* slab size of the device pool; a multiple
                                   of 16 bytes (INVALID otherwise)                             */
  uint64_t host_slab_bytes;     /* slab size of the host pool (multiple of 16 bytes)          */
  uint64_t stage_ring_bytes;    /* pinned Stage Buffer for weights (2 GB)      */
  uint64_t stage_chunk_bytes;   /* weight pipeline chunk                                      */
  uint64_t staging_slot_bytes;  /* device staging slot for KV gather/scatter                  */
  uint64_t table_arena_bytes;   /* device block-table arena                                   */
  int32_t dev_slab_layout;      /* AEG_LAYER_MAJOR | AEG_BLOCK_MAJOR                          */
  int32_t host_slab_layout;
  int32_t staging_slots;        /* slots per direction                                        */
  int32_t host_threads;         /* weight-staging copy threads                                */
  int32_t kernel;               /* AEG_KERNEL_*                                               */
  int32_t migrate_ctas;         /* CTAs used by the NVLink migrate kernel (SM budget), 0=auto */
  uint32_t flags;               /* AEG_CFG_*                                                  */
  int32_t numa_node;            /* pinned host memory placement: 0 = the GPU's NUMA node (from
                                   sysfs; unbound if unknown), n > 0 = node n-1, -1 = no binding */
  uint32_t dma_piece_mib;       /* swap-out D2H piece (MiB) for sub-layer rule-❷ waits of a
                                   chained swap-in; 0 = 128, >= 4096 = one piece
                                   per segment (per-layer events only).  Pieces are cut at host-run
                                   boundaries; very small pieces on big transfers can exceed the
                                   ~1,000 pending copies a stream holds, and the data call then
                                   blocks until the copy engine drains (correct, not async)      */
  uint32_t pack_layer_mib;      /* KV swaps: layers smaller than this share one staging segment
                                   (one kernel launch, fewer copy commands, readiness per
                                   segment), keeping >= 4 segments per transfer (fewer layers:
                                   one per segment); 0 = the default             */
  uint32_t reserved[4];
} aeg_config;

/* One checkpoint tensor in the (pageable or registered) host Model Cache, row-major
 * [rows, cols] of elem_bytes.  `layer` is the caller's readiness index (>= 0): the transfer's
 * layer-l event fires when every tensor with that index has landed.  `groups` > 1 splits
 * fused tensors (e.g. QKV) per group before taking the rank's part (COL/VOCAB only). */
typedef struct {
  const void* host_src;
  uint64_t rows, cols;
  int32_t elem_bytes, layer, split, groups;
} aeg_weight_desc;

typedef struct {
  aeg_kv_shape shape;
  uint64_t slabs, owned_blocks, quarantined_blocks;
} aeg_shape_stats;

typedef struct {
  uint64_t pool_bytes, slab_bytes, n_slabs, free_slabs;
  uint64_t owned_blocks, quarantined_blocks;
  uint64_t used_bytes;          /* owned blocks x block bytes                                */
  uint64_t assigned_bytes;      /* slabs assigned to a shape x slab bytes                    */
  uint64_t peak_used_bytes, peak_assigned_bytes;
  int32_t n_shapes;             /* entries filled in per_shape (<= 16)                       */
  int32_t pad;
  aeg_shape_stats per_shape[16];
} aeg_pool_stats;

/* ---- lifecycle -------------------------------------------------------------------------- */

/* Fill *cfg with defaults: 1 GiB slabs (layer-major), 2 GiB stage ring of 64 MiB chunks,
 * 3 x 1 GiB staging slots per direction, 8 host threads, AUTO kernels; region sizes 0 (a zero
 * device_kv_bytes is sized at aeg_init from 90% of free VRAM, reading 22; zero host KV / weights
 * regions are empty).  Returns AEG_OK (INVALID if cfg is NULL). */
int aeg_config_default(aeg_config* cfg);

/* Create a context on CUDA device `device`: one cudaMalloc for [KV | weights | staging |
 * tables] ("in one allocation") and one pinned host allocation for the CPU
 * KV cache and Stage Buffer, pinned once.  With AEG_CFG_HOST_ONLY no CUDA
 * call is made and `device` is ignored.  Errors: INVALID (bad config), CUDA, OOM. */
int aeg_init(int device, const aeg_config* cfg, aeg_ctx* out);

/* Wait for all transfers, stop the daemon, free everything.  NULL is accepted. */
int aeg_shutdown(aeg_ctx ctx);

/* Thread-local text of the last error on this thread ("" if none).  Never NULL. */
const char* aeg_last_error(void);

/* ---- unified KV cache (H1) ---------------------------------------------------------------- */

/* Allocate n blocks of `shape` from pool: free non-quarantined blocks of
 * same-shape slabs (lowest slab, lowest index first), then new slabs (lowest first).  Runs the
 * daemon's reclaim step first.  All-or-nothing: on AEG_ERR_OOM nothing is allocated.
 * out[n] receives the handles in allocation order.  n == 0 is a no-op. */
int aeg_kv_alloc(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, int32_t n, aeg_block* out);

/* Free n owned blocks of pool.  Blocks still read or written by an
 * incomplete transfer go to the move list and are reclaimed by the daemon (step ⑧).  An empty
 * slab returns to the unassigned state.  All handles are validated first: INVALID for handles
 * of another pool / outside any assigned slab, STATE for unowned or repeated handles; on error
 * nothing is freed. */
int aeg_kv_free(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n);

/* Step ⑧ on demand (§5.3: "a daemon thread periodically queries
 * (cudaEventQuery) events in the move lists to reclaim the blocks once the transfers complete"):
 * release move-list blocks whose transfers completed, reap released transfers.  blocking != 0
 * first waits for every in-flight transfer.  Returns AEG_OK. */
int aeg_reclaim(aeg_ctx ctx, int blocking);

/* Pool statistics.  Fig. 16's fragmentation, "the ratio of unused memory to peak allocated memory"
 * (PAPER.md:2030-2033), is (assigned_bytes - used_bytes) / peak_assigned_bytes. */
int aeg_stats(aeg_ctx ctx, int32_t pool, aeg_pool_stats* out);

/* Decode a handle.  Any output pointer may be NULL. */
int aeg_block_info(aeg_ctx ctx, aeg_block b, int32_t* pool, uint32_t* slab, uint32_t* index);

/* Address of layer `layer` of block b inside its slab (§5.2: a slab "serving as
 * a pool of KV cache blocks for that specific shape"; the in-slab layout is reading 5): device
 * pointer (device pool) or host pointer (host pool, pinned and device-mapped).  The block must be
 * owned and of `shape`; INVALID otherwise.  *p is written only on AEG_OK. */
int aeg_block_ptr(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, aeg_block b,
                  int32_t layer, void** p);

/* Block table for a consumer (e.g. a PagedAttention kernel): off0[i] = byte offset of layer 0 of
 * blocks[i] from the pool base, and *layer_stride = bytes between consecutive layers of a block (the
 * same for every block of `shape` in this pool), so layer l of block i is at base + off0[i] +
 * l * layer_stride.  All blocks must be owned and of `shape`.  O(n), one call. */
int aeg_block_offsets(aeg_ctx ctx, int32_t pool, const aeg_kv_shape* shape, const aeg_block* blocks,
                      int32_t n, uint64_t* off0, uint64_t* layer_stride);

/* Base pointer and size of a pool's region (device pointer for DEVICE, host pointer for HOST). */
int aeg_pool_region(aeg_ctx ctx, int32_t pool, void** base, uint64_t* bytes);

/* Base pointer (valid in this process: UVA / CUDA-IPC mapping) and size of the device KV region of
 * an imported peer (aeg_import_peer index `peer`), for callers that address the peer's blocks
 * themselves (e.g. a copy-engine comparison route).  AEG_ERR_INVALID if the peer was not imported. */
int aeg_peer_region(aeg_ctx ctx, int32_t peer, void** base, uint64_t* bytes);

/* ---- KV movement (H2-H6) ------------------------------------------------------------------ */

/* Swap-out P->C (Fig. 10 steps ①②): for i < n and every layer l,
 * host[addr_H(host[i], l) .. + Cl) = dev[addr_D(dev[i], l) .. + Cl).  Per layer: gather kernel
 * (paged -> contiguous device staging slot) then copy-engine D2H per contiguous host run, then
 * ev[l] is recorded.  Rule ❷: layer l of block b waits for b's last writer's ev[l]; rule ❸: the
 * writes into host blocks wait for their last readers/writers.  Both tables hold owned blocks of
 * `shape`; dev handles must be distinct, host handles must be distinct.  AEG_FREE_SRC frees the
 * device blocks (move list until done).  *out receives the transfer (L = num_layers events). */
int aeg_kv_swap_out(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* dev,
                    const aeg_block* host, int32_t n, uint32_t flags, aeg_xfer* out);

/* Swap-in C->D (steps ③④⑤): dev[addr_D(dev[i], l)] = host[addr_H(host[i], l)]
 * for every layer; per layer: copy-engine H2D per host run into a staging slot, scatter kernel into
 * the device blocks, ev[l].  The H2D of layer l waits on the last writer of the host blocks'
 * ev[l] (rule ❷ per layer, reading 12).  AEG_FREE_SRC frees the host blocks. */
int aeg_kv_swap_in(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* host,
                   const aeg_block* dev, int32_t n, uint32_t flags, aeg_xfer* out);

/* Prefill->decode hand-off (north star; Fig. 10, the KV of a request moving from
 * a prefill instance to a decoding instance, here directly GPU-to-GPU instead of through the CPU
 * cache): dst_pool_of(peer)[addr_dst(dst[i], l)] = dev[addr_src(src[i], l)] for
 * every layer, by a fused kernel on this GPU that reads local blocks and stores 16-byte vectors
 * straight into the peer's pool over NVLink/NVSwitch (no staging).  `peer` is an index given to
 * aeg_import_peer, or -1 for this context's own device pool (local relocation).  dst handles are
 * allocated by the peer in its device pool and are trusted (validated against the peer's
 * geometry only).  Per-layer events are interprocess-capable; export them with aeg_xfer_export.
 * Consecutive layers share a kernel launch up to ~1 ms of copying (4 GiB on one GPU, 512 MiB to
 * another GPU); each layer's event is recorded when the launch holding it completes.
 * AEG_FREE_SRC frees the source blocks.  AEG_MIGRATE_CE takes the copy-engine route (SURVEY H5
 * alternative): per staging segment a gather kernel packs the source blocks into the out staging
 * ring, then copy engines write the destination runs (one command per run and layer, or one 2-D
 * command per layer across equal whole runs); the decode GPU's SMs are never used and the source
 * GPU's only for the HBM-speed gather.  Same bytes, same events, same rules. */
int aeg_kv_migrate(aeg_ctx ctx, const aeg_kv_shape* shape, const aeg_block* src, int32_t peer,
                   const aeg_block* dst, int32_t n, uint32_t flags, aeg_xfer* out);

/* Paper route P->C->D (Fig. 10 ③④⑤; NEXT-2): swap-in from ANOTHER process's
 * shared CPU KV region (the peer exported with AEG_CFG_SHARED_HOST; `peer` as given to
 * aeg_import_peer, or -1 for this context's own host pool).  Layer l's H2D waits on layer l of
 * transfer `after` (0 = none) — typically the peer's swap-out imported with aeg_xfer_import (rule ❷
 * across instances via IPC events).  peer_host handles are validated against
 * the peer's geometry only; ownership stays with the peer, which frees them with aeg_kv_free_after
 * on this transfer (rule ❸).  Otherwise as aeg_kv_swap_in (AEG_FREE_SRC is INVALID for a peer). */
int aeg_kv_swap_in_from(aeg_ctx ctx, const aeg_kv_shape* shape, int32_t peer, const aeg_block* peer_host,
                        const aeg_block* dev, int32_t n, aeg_xfer after, uint32_t flags, aeg_xfer* out);

/* Free owned blocks that a transfer `after` (local or imported) still reads or writes: they go to
 * the move list until `after` completes (step ⑧), e.g. the prefill instance's
 * CPU blocks after the decode instance's swap-in of them was imported. */
int aeg_kv_free_after(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n, aeg_xfer after);

/* Order every later transfer of this context after the work currently enqueued on `cuda_stream`
 * (a cudaStream_t; NULL = legacy default stream), e.g. the prefill kernels that wrote the blocks. */
int aeg_stream_fence(aeg_ctx ctx, void* cuda_stream);

/* Rule ❶ (Table 2): readiness of layer `layer` of transfer x.
 *   QUERY       -> AEG_OK when complete, AEG_NOT_READY otherwise (never blocks)
 *   WAIT_STREAM -> work submitted to `cuda_stream` afterwards runs after the layer landed
 *   BLOCK       -> returns when the layer landed
 * `layer` = -1 means the whole transfer.  Once ready, a layer stays ready.  STATE for an unknown
 * or released transfer, INVALID for a layer out of range. */
int aeg_layer_ready(aeg_ctx ctx, aeg_xfer x, int32_t layer, int32_t mode, void* cuda_stream);

/* Number of readiness layers of x. */
int aeg_xfer_layers(aeg_ctx ctx, aeg_xfer x, int32_t* layers);

/* The caller will not query x again; its CUDA events (Table 2) are recycled
 * once it completes (and, for a transfer imported by another context of this process, once that
 * import is reaped).  STATE for an unknown transfer. */
int aeg_xfer_release(aeg_ctx ctx, aeg_xfer x);

/* ---- weights (H7, N1) ----------------------------------------------------------------------- */

/* Stage n tensors of the Model Cache into the weights region: each tensor's
 * rank-`tp_rank` shard (of tp_size) is bump-allocated at off_{k+1} = align256(off_k + |shard_k|)
 * and copied host threads -> pinned Stage Buffer ring -> copy-engine H2D in
 * stage_chunk_bytes chunks.  Padding between shards is written as zeros.  If a tensor lies in a
 * region registered with aeg_host_register it is DMA'd directly (2-D copy for ROW shards).
 * dev_offsets_out[n] receives byte offsets inside the weights region.  Returns after the host
 * pipeline is started; the layer events are recorded as chunks are issued (WAIT_STREAM and
 * BLOCK readiness first wait on the host until the event is recorded).
 * Composition note (measured): one copy engine serves a busy H2D stream until it
 * drains, so in a model switch enqueue the incoming KV swap-in BEFORE the weights, or the KV lands
 * after the whole model.
 * INVALID for non-divisible splits, OOM if the region is exhausted. */
int aeg_weights_stage(aeg_ctx ctx, const aeg_weight_desc* descs, int32_t n, int32_t tp_rank,
                      int32_t tp_size, uint64_t* dev_offsets_out, aeg_xfer* out);

/* Reset the bump pointer to `offset` (0 = region base): "deallocations can be done instantly by
 * simply resetting that pointer".  Does not wait: later staging and
 * relocation run on the same weights stream, so they are ordered after earlier ones.  INVALID for
 * an offset beyond the region or not 256-byte aligned. */
int aeg_weights_reset(aeg_ctx ctx, uint64_t offset);

/* Current bump pointer, base pointer and size of the weights region. */
int aeg_weights_region(aeg_ctx ctx, void** base, uint64_t* bytes, uint64_t* bump);

/* N1 (Fig. 9 step 3.b): move `bytes` of the weights region from src_off to
 * dst_off (memmove semantics, overlap-safe) on the device, as one transfer with one layer. */
int aeg_weights_relocate(aeg_ctx ctx, uint64_t src_off, uint64_t dst_off, uint64_t bytes,
                         aeg_xfer* out);

/* Weight-pipeline counters since init: chunks issued, host milliseconds the issuer waited for host
 * fills (fill-bound), and summed milliseconds fill tasks waited for a Stage Buffer slot's previous
 * DMA (PCIe-bound).  Any output pointer may be NULL. */
int aeg_weights_stats(aeg_ctx ctx, uint64_t* chunks, double* issuer_wait_fill_ms, double* fill_wait_slot_ms);

/* Page-lock an existing host range (e.g. a Model Cache) so weights in it DMA directly. */
int aeg_host_register(aeg_ctx ctx, void* ptr, uint64_t bytes);
int aeg_host_unregister(aeg_ctx ctx, void* ptr);

/* ---- multi-process (H5) ------------------------------------------------------------------- */

/* Serialise this context's device-pool IPC handle, geometry and interprocess event ring into
 * buf (capacity *len in, bytes used out).  buf == NULL: *len receives the required size.
 * PAPER.md:1528-1532 §5.3 ("Events are also passed between instances via interprocess
 * communication (IPC) for synchronizing different instances"; cudaIpcGetEventHandle, Table 2). */
int aeg_export_ipc(aeg_ctx ctx, void* buf, uint64_t* len);

/* Map a peer's device pool (cudaIpcOpenMemHandle, or a direct pointer when the peer lives in
 * this process) and its event ring (cudaIpcOpenEventHandle, Table 2), and
 * enable peer access when the peer is another GPU.  `peer` is the caller's index for it (0..63);
 * importing an index again replaces that peer's mappings.  INVALID for a malformed blob or index,
 * STATE in a host-only context, CUDA when the mapping or peer access fails. */
int aeg_import_peer(aeg_ctx ctx, int32_t peer, const void* buf, uint64_t len);

/* Serialise transfer x's per-layer interprocess events (after it was enqueued) so the peer can
 * wait on them; aeg_xfer_import turns such a blob into a local transfer id of the importer.  A
 * swap-out whose D2H ran in pieces (aeg_config.dma_piece_mib) also exports its per-(layer, piece)
 * events, piece table and written host handles, so a peer's aeg_kv_swap_in_from(after = it) waits
 * per piece (sub-layer rule ❷ across instances).  Call with buf = NULL to get the size.
 * Lifetime: export before aeg_xfer_release (AEG_ERR_STATE after).  Another process opens the events
 * by IPC handle and owns those.  A context in the SAME process borrows the exporter's events: the
 * exporter keeps the transfer (does not recycle its events) until every such import has been
 * released and reaped, and the exporting context must be shut down after its importers. */
int aeg_xfer_export(aeg_ctx ctx, aeg_xfer x, void* buf, uint64_t* len);
int aeg_xfer_import(aeg_ctx ctx, int32_t peer, const void* buf, uint64_t len, aeg_xfer* out);

/* SM budget of later aeg_kv_migrate launches (aeg_config.migrate_ctas at run time): ctas > 0 caps
 * the migrate kernel's grid at `ctas` CTAs of 256 threads (the block scheduler spreads them one per
 * SM first, so ctas <= 148 ~ that many SMs), leaving the rest of the GPU to the decode instance's
 * compute; 0 = a full wave.  AEG_ERR_INVALID if ctas < 0.  Transfers already enqueued keep theirs. */
int aeg_set_migrate_ctas(aeg_ctx ctx, int32_t ctas);

/* ---- instrumentation ---------------------------------------------------------------------- */

/* Kernel counters since the last reset (needs AEG_CFG_TIMING for ms): kind 0 gather, 1 scatter,
 * 2 migrate, 3 relocate, 4 block-table fetch (3 and 4: launches and bytes only, never timed).
 * launches / algorithmic bytes moved (payload read + written) / summed CUDA-event ms of the
 * launches (each timed on its own stream). */
int aeg_kernel_stats(aeg_ctx ctx, int32_t kind, uint64_t* launches, uint64_t* bytes, double* ms);
int aeg_kernel_stats_reset(aeg_ctx ctx);

/* Record the Table 2 primitive log (record / wait / op reads+writes / sync) for the rule checker
 * (oracle/rules.py).  Only for small tests: every block-layer cell is logged. */
int aeg_trace_enable(aeg_ctx ctx, int on);
/* Copy out (and clear) the trace as text lines; *len in = capacity, out = bytes written.  If the
 * buffer is too small, *len receives the required size and AEG_ERR_INVALID is returned. */
int aeg_trace_read(aeg_ctx ctx, char* buf, uint64_t* len);

/* Test hooks for AEG_CFG_HOST_ONLY contexts: a synthetic transfer touching `blocks` of `pool`
 * (blocks freed meanwhile go to the move list) and its completion. */
int aeg_debug_xfer_begin(aeg_ctx ctx, int32_t pool, const aeg_block* blocks, int32_t n,
                         aeg_xfer* out);
int aeg_debug_xfer_complete(aeg_ctx ctx, aeg_xfer x);

#ifdef __cplusplus
}
#endif
#endif /* AEG_H_ */
