// KV movement (H2-H6): swap-out (gather kernel -> copy-engine D2H), swap-in (copy-engine H2D ->
// scatter kernel), NVLink migrate (fused gather -> remote store) and weight relocation (N1).
//
// Every transfer is enqueued entirely from the calling thread, so all its events are recorded
// before the call returns.  Stream roles (Fig. 10 "KV-Out" / "KV-In" streams):
//   swap-out : s_gather (kernel, high priority)  ->  s_d2h     (copy engine)
//   swap-in  : s_h2d    (copy engine)            ->  s_scatter (kernel, high priority)
// The two halves of a direction hand staging slots back and forth with full/free events.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "engine.h"

// Layers per local hand-off launch, in MiB (see Ctx::migrate); overridable for experiments
// (tools/gpu_migrate_pack.sh builds with -DAEG_MIGRATE_LOCAL_PACK_MIB=...).
#ifndef AEG_MIGRATE_LOCAL_PACK_MIB
#define AEG_MIGRATE_LOCAL_PACK_MIB 4096
#endif

namespace aeg {

namespace {

struct Seg {
  int32_t la, lb, i0, i1;
};

// A transfer of n blocks x L layers is cut into segments that fit one staging slot: whole layers
// (several when a layer is smaller than pack_bytes, aeg_config.pack_layer_mib) or, for big layers,
// runs of blocks of one layer.  Segments are in layer order, so the per-layer event can be recorded
// right after a layer's last segment.  Packing keeps at least kMinSegments segments: the two copy
// engines overlap only across segments (the swap-in's H2D of one segment runs while the swap-out's
// D2H of the next does), so a transfer packed into one segment has no duplex overlap at all —
// configs[0]'s 2-layer round trip took 172 us as one segment, 147 us as two (bench `c1`).
constexpr int32_t kMinSegments = 4;
std::vector<Seg> plan(int32_t L, int32_t n, uint64_t chunk, uint64_t slot_bytes, uint64_t pack_bytes) {
  std::vector<Seg> out;
  if (n == 0) return out;
  const uint64_t layer = uint64_t(n) * chunk;
  if (layer <= slot_bytes) {
    int32_t lps = 1;
    if (layer < pack_bytes)
      lps = int32_t(std::max<uint64_t>(1, std::min<uint64_t>(pack_bytes, slot_bytes) / layer));
    lps = std::min(lps, std::max<int32_t>(1, L / kMinSegments));
    for (int32_t la = 0; la < L; la += lps) out.push_back({la, std::min(L, la + lps), 0, n});
  } else {
    // balanced runs of blocks (no small tail segment): ceil(n / cap) segments of near-equal size
    const int32_t cap = int32_t(slot_bytes / chunk);
    const int32_t nseg = (n + cap - 1) / cap;
    for (int32_t l = 0; l < L; ++l)
      for (int32_t q = 0; q < nseg; ++q)
        out.push_back({l, l + 1, int32_t(int64_t(n) * q / nseg), int32_t(int64_t(n) * (q + 1) / nseg)});
  }
  return out;
}

// Maximal runs of host handles that are consecutive blocks of one slab.
struct Run {
  int32_t i0, m;
  aeg_block first;
};
std::vector<Run> runs_of(const aeg_block* h, int32_t n) {
  std::vector<Run> r;
  for (int32_t i = 0; i < n;) {
    int32_t m = 1;
    while (i + m < n && block_slab(h[i + m]) == block_slab(h[i]) && block_idx(h[i + m]) == block_idx(h[i]) + uint32_t(m))
      ++m;
    r.push_back({i, m, h[i]});
    i += m;
  }
  return r;
}

// Trace cells of a staging-ring range (16 KiB granules), so the rule checker sees ring reuse.
std::string ring_cells(const char* tag, uint64_t off, uint64_t size) {
  std::string s;
  for (uint64_t g = off >> 14; g < (off + size + (1u << 14) - 1) >> 14; ++g) {
    if (!s.empty()) s += ',';
    s += tag;
    s += ':';
    s += std::to_string(g);
  }
  return s;
}

std::vector<uint64_t> uniq(std::vector<uint64_t> v) {
  std::sort(v.begin(), v.end());
  v.erase(std::unique(v.begin(), v.end()), v.end());
  return v;
}

// Block-range pieces [a, b) of a segment for its host DMAs (sub-layer rule-❷ events, Xfer::pev).
// A single-layer segment larger than piece_bytes is cut at host-run boundaries (maximal runs of
// consecutive host blocks of one slab), grouping whole runs up to piece_bytes, so each piece stays
// ONE copy-engine command where host_dmas can merge it (equal whole runs at a constant pitch): a
// stream holds only ~1,000 pending copies before the enqueueing call blocks
// (tools/queue_depth_probe.py), and balanced cuts through runs tripled the command count.  A run
// longer than piece_bytes is split evenly.  A multi-layer (packed) segment stays one piece.
std::vector<std::pair<int32_t, int32_t>> pieces_of(const Seg& g, uint64_t chunk, uint64_t piece_bytes,
                                                   const std::vector<Run>& runs) {
  std::vector<std::pair<int32_t, int32_t>> out;
  if (g.lb - g.la != 1 || uint64_t(g.i1 - g.i0) * chunk <= piece_bytes) {
    out.push_back({g.i0, g.i1});
    return out;
  }
  const int32_t cap = int32_t(std::max<uint64_t>(1, piece_bytes / chunk));  // blocks per piece
  int32_t a = g.i0;
  for (const Run& r : runs) {
    const int32_t s0 = std::max(r.i0, g.i0), e0 = std::min(r.i0 + r.m, g.i1);
    if (s0 >= e0) continue;
    if (e0 - s0 > cap) {  // a long run: close the open piece, split the run evenly
      if (s0 > a) out.push_back({a, s0});
      const int32_t np = (e0 - s0 + cap - 1) / cap;
      for (int32_t q = 0; q < np; ++q)
        out.push_back({s0 + int32_t(int64_t(e0 - s0) * q / np), s0 + int32_t(int64_t(e0 - s0) * (q + 1) / np)});
      a = e0;
      continue;
    }
    if (e0 - a > cap && s0 > a) {  // this run would overfill the open piece: close it before the run
      out.push_back({a, s0});
      a = s0;
    }
  }
  if (a < g.i1) out.push_back({a, g.i1});
  return out;
}

}  // namespace

// Largest pitch a 2-D copy accepts (cudaDevAttrMaxPitch, 2^31-1 on B200), queried once.  Runs in
// slabs further apart than this (e.g. whole 1 GiB slabs 0, 2, 4 -> pitch 2 GiB) are not merged.
static int64_t max_pitch() {
  static const int64_t v = [] {
    int dev = 0, mp = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&mp, cudaDevAttrMaxPitch, dev) != cudaSuccess ||
        mp <= 0)
      return int64_t(INT32_MAX);
    return int64_t(mp);
  }();
  return v;
}

// Copy-engine DMAs between a staging slot and the host blocks of segment g (layer-major staging
// image inside the slot).  dir = cudaMemcpyDeviceToHost (swap-out) or HostToDevice (swap-in).
// `hp` / `hbase` is the pool on the far side of the copy engine: this context's host pool (D2H / H2D)
// or, for the copy-engine hand-off route, a device pool (this one's or a peer's; kind = Default).
// to_pool: staging -> pool (swap-out, hand-off) or pool -> staging (swap-in).
static void host_dmas(const SlabPool& hp, char* hbase, const Shape& sh, const std::vector<Run>& runs, const Seg& g,
                      char* slot, bool to_pool, cudaMemcpyKind dir, cudaStream_t s) {
  const uint64_t Cl = sh.chunk(), hstride = hp.lstride(sh);
  const int32_t nseg = g.i1 - g.i0, nl = g.lb - g.la;
  if (hp.layout == AEG_LAYER_MAJOR) {
    // Within one layer, runs of equal length whose host addresses step by a constant pitch
    // (typically whole slabs: k blocks, pitch S) become ONE 2-D copy.  The grouping is the same in
    // every layer (layers differ by a constant offset), so a segment costs nl x groups copies this
    // way, or one copy per run (2-D over its nl layers) the other way: take the fewer commands.
    struct Group {
      int32_t a0, m;
      size_t rows;
      int64_t pitch;
      aeg_block first;  // host block of the group's first row at index a0
    };
    std::vector<Group> groups;
    size_t nruns = 0;
    auto host_of = [&](aeg_block first_of_run, int32_t run_i0, int32_t a, int32_t l) {
      const aeg_block hb = make_block(AEG_POOL_HOST, block_slab(first_of_run), block_idx(first_of_run) + uint32_t(a - run_i0));
      return hbase + hp.off0(hb, sh) + uint64_t(l) * hstride;
    };
    size_t q = 0;
    while (q < runs.size()) {
      const Run& r0 = runs[q];
      const int32_t a0 = std::max(r0.i0, g.i0), b0 = std::min(r0.i0 + r0.m, g.i1);
      if (a0 >= b0) {
        ++q;
        continue;
      }
      const int32_t m = b0 - a0;
      size_t e = q + 1;
      int64_t pitch = 0;
      char* prev = host_of(r0.first, r0.i0, a0, g.la);
      while (e < runs.size()) {  // extend while the next run is whole, same length, same pitch
        const Run& r = runs[e];
        if (r.i0 < g.i0 || r.i0 + r.m > g.i1 || r.m != m || r.i0 != a0 + int32_t(e - q) * m) break;
        char* cur = host_of(r.first, r.i0, r.i0, g.la);
        const int64_t p = cur - prev;
        if (e == q + 1) pitch = p;
        if (p != pitch || p < int64_t(m) * int64_t(Cl) || p > max_pitch()) break;
        prev = cur;
        ++e;
      }
      groups.push_back({a0, m, e - q, pitch,
                        make_block(AEG_POOL_HOST, block_slab(r0.first), block_idx(r0.first) + uint32_t(a0 - r0.i0))});
      nruns += e - q;
      q = e;
    }
    if (nl == 1 || uint64_t(nl) * groups.size() < nruns) {
      for (int32_t t = 0; t < nl; ++t)
        for (const Group& gr : groups) {
          char* h0 = hbase + hp.off0(gr.first, sh) + uint64_t(g.la + t) * hstride;
          char* st0 = slot + (uint64_t(t) * nseg + uint64_t(gr.a0 - g.i0)) * Cl;
          const uint64_t w = uint64_t(gr.m) * Cl;
          if (gr.rows == 1) {
            if (to_pool)
              CUDA_TRY(cudaMemcpyAsync(h0, st0, w, dir, s));
            else
              CUDA_TRY(cudaMemcpyAsync(st0, h0, w, dir, s));
          } else if (to_pool) {
            CUDA_TRY(cudaMemcpy2DAsync(h0, size_t(gr.pitch), st0, w, w, gr.rows, dir, s));
          } else {
            CUDA_TRY(cudaMemcpy2DAsync(st0, w, h0, size_t(gr.pitch), w, gr.rows, dir, s));
          }
        }
      return;
    }
  }
  for (const Run& r : runs) {
    const int32_t a = std::max(r.i0, g.i0), b = std::min(r.i0 + r.m, g.i1);
    if (a >= b) continue;
    const aeg_block hb = make_block(AEG_POOL_HOST, block_slab(r.first), block_idx(r.first) + uint32_t(a - r.i0));
    const int32_t m = b - a;
    char* host0 = hbase + hp.off0(hb, sh) + uint64_t(g.la) * hstride;
    char* st0 = slot + uint64_t(a - g.i0) * Cl;
    const uint64_t st_pitch = uint64_t(nseg) * Cl;  // next layer inside the slot
    if (hp.layout == AEG_LAYER_MAJOR) {
      // the run is contiguous within each layer: one 1-D copy, or one 2-D copy over the layers
      const uint64_t w = uint64_t(m) * Cl;
      if (nl == 1 || int64_t(hstride) > max_pitch()) {
        for (int32_t t = 0; t < nl; ++t) {
          char* h = host0 + uint64_t(t) * hstride;
          char* st = st0 + uint64_t(t) * st_pitch;
          if (to_pool)
            CUDA_TRY(cudaMemcpyAsync(h, st, w, dir, s));
          else
            CUDA_TRY(cudaMemcpyAsync(st, h, w, dir, s));
        }
      } else if (to_pool) {
        CUDA_TRY(cudaMemcpy2DAsync(host0, hstride, st0, st_pitch, w, nl, dir, s));
      } else {
        CUDA_TRY(cudaMemcpy2DAsync(st0, st_pitch, host0, hstride, w, nl, dir, s));
      }
    } else {
      // block-major: within a layer consecutive blocks are L*Cl apart -> one 2-D copy per layer
      for (int32_t t = 0; t < nl; ++t) {
        char* h = host0 + uint64_t(t) * hstride;
        char* st = st0 + uint64_t(t) * st_pitch;
        if (to_pool)
          CUDA_TRY(cudaMemcpy2DAsync(h, sh.block(), st, Cl, Cl, m, dir, s));
        else
          CUDA_TRY(cudaMemcpy2DAsync(st, Cl, h, sh.block(), Cl, m, dir, s));
      }
    }
  }
}

// Under AUTO every gather/scatter above 2 KiB chunks uses BULKW (cp.async.bulk issued by 6 warps per
// CTA).  Stores into another GPU's pool use LSU under AUTO (plain st.global to peer addresses).
#define ipc_events(flags) (((flags) & AEG_IPC_EVENTS) || (cfg.flags & AEG_CFG_SHARED_HOST))

// AUTO by chunk size, from tools/small_chunk_probe.cu (profiles/r02/small_chunk_probe_final_bulkw.txt, 1 GiB
// gather / scatter launches over 30 GB-spread tables, median TB/s) and the bench's own C2 step:
//   2 KiB: WARP 5.97 / 6.08, BULKW 5.47 / 5.51, LSU 1.8, BULK 0.8
//   4 KiB: BULKW 5.98 / 5.93, WARP 5.56 / 5.63, LSU 3.4-3.5
//   8 KiB: BULKW 6.26 / 6.36, WARP 5.74, LSU 5.48, BULK 2.99
//   16-32 KiB: BULKW 6.33-6.47, LSU 5.8-6.1, BULK 5.1-6.1;  256 KiB: BULKW 6.47 / 6.44, BULK 6.1
//   C2 step in-step (256 KiB chunks, 1 GiB launches next to PCIe DMA): BULKW 5.91 / 5.81 TB/s
//   gather / scatter vs BULK 5.73 / 5.53 (profiles/r02/bench_bulkw_vs_bulk.txt)
static int impl_of(const aeg_config& cfg, uint64_t chunk) {
  if (cfg.kernel == AEG_KERNEL_LSU) return IMPL_LSU;
  if (cfg.kernel == AEG_KERNEL_BULK) return IMPL_BULK;
  if (cfg.kernel == AEG_KERNEL_WARP) return IMPL_WARP;
  if (cfg.kernel == AEG_KERNEL_BULKW) return IMPL_BULKW;
  return chunk <= (2u << 10) ? IMPL_WARP : IMPL_BULKW;
}

// Optional host-side phase timer of swap_out (AEG_HOST_PROFILE=1: totals printed at exit): where
// the enqueue time of a call goes (validation, rule bookkeeping, table, segments, notes, free).
namespace {
struct HostProf {
  bool on = getenv("AEG_HOST_PROFILE") != nullptr;
  double t[8] = {0};
  uint64_t calls = 0;
  ~HostProf() {
    if (on && calls)
      fprintf(stderr, "[aeg host profile] swap_out x%llu, us per call: validate %.1f deps %.1f table %.1f "
              "plan %.1f segments %.1f record %.1f notes %.1f free %.1f\n", (unsigned long long)calls,
              t[0] / calls, t[1] / calls, t[2] / calls, t[3] / calls, t[4] / calls, t[5] / calls, t[6] / calls,
              t[7] / calls);
  }
} g_prof;
struct PhaseClock {
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
  void lap(int i) {
    if (!g_prof.on) return;
    auto t1 = std::chrono::steady_clock::now();
    g_prof.t[i] += std::chrono::duration<double, std::micro>(t1 - t0).count();
    t0 = t1;
  }
};
}  // namespace

// ----------------------------------------------------------------------------- swap-out H3
uint64_t Ctx::swap_out(const Shape& sh, const aeg_block* dev, const aeg_block* host, int32_t n, uint32_t flags) {
  AEG_REQUIRE(!host_only, AEG_ERR_STATE, "host-only context has no data path");
  SlabPool &dp = pool[AEG_POOL_DEVICE], &hp = pool[AEG_POOL_HOST];
  PhaseClock pc;
  if (g_prof.on) g_prof.calls++;
  dp.check_owned(dev, n, &sh);
  hp.check_owned(host, n, &sh);
  AEG_REQUIRE(sh.chunk() <= ring_out.slot_bytes, AEG_ERR_INVALID, "chunk larger than a staging slot");
  Xfer* x = new_xfer(X_SWAP_OUT, sh.L, ipc_events(flags));
  pc.lap(0);
  std::vector<uint64_t> rdeps, wdeps;
  if (!(flags & AEG_NO_DEPS)) {
    for (int32_t i = 0; i < n; ++i) dp.deps_for_read(dev[i], rdeps);
    for (int32_t i = 0; i < n; ++i) hp.deps_for_write(host[i], wdeps);
  }
  rdeps = uniq(rdeps);
  wdeps = uniq(wdeps);
  pc.lap(1);
  char *htab = nullptr, *dtab = nullptr;
  if (n > 0) {
    alloc_table(uint64_t(n) * 8, x->id, &htab, &dtab);
    uint64_t* t = reinterpret_cast<uint64_t*>(htab);
    for (int32_t i = 0; i < n; ++i) t[i] = dp.off0(dev[i], sh);
    fetch_table(dtab, htab, uint64_t(n) * 8, s_gather);
  }
  pc.lap(2);
  const auto segs = plan(sh.L, n, sh.chunk(), ring_out.slot_bytes, uint64_t(cfg.pack_layer_mib) << 20);
  const auto runs = runs_of(host, n);
  const uint64_t dstride = dp.lstride(sh);
  const uint64_t piece_bytes = uint64_t(cfg.dma_piece_mib) << 20;
  // sub-layer D2H pieces: the same block ranges in every layer (segments repeat per layer)
  for (const Seg& g : segs) {
    if (g.la != 0) break;
    if (g.lb != 1) break;  // packed small layers: per-layer events only
    for (auto& pc : pieces_of(g, sh.chunk(), piece_bytes, runs)) x->piece_lo.push_back(pc.first);
  }
  if (x->piece_lo.size() > 1) {
    x->npiece = int32_t(x->piece_lo.size());
    x->piece_lo.push_back(n);
    x->pev.resize(size_t(sh.L) * size_t(x->npiece));
    for (auto& e : x->pev) e = take_event(x->ipc);  // exportable with the layer events
    x->wpos.reserve(size_t(n) * 2);
    for (int32_t i = 0; i < n; ++i) x->wpos.emplace(host[i], i);
  } else {
    x->piece_lo.clear();
  }
  pc.lap(3);
  int32_t pidx = 0;
  for (const Seg& g : segs) {
    if (g.i0 == 0) pidx = 0;
    if (g.i0 == 0) wait_deps(s_gather, rdeps, g.la, g.lb);  // rule ❷
    cudaEvent_t full, freed;
    uint64_t roff;
    std::vector<cudaEvent_t> waited;
    const uint64_t seg_bytes = uint64_t(g.lb - g.la) * uint64_t(g.i1 - g.i0) * sh.chunk();
    char* sp = ring_out.acquire(seg_bytes, s_gather, &full, &freed, &roff, tracing ? &waited : nullptr);
    for (cudaEvent_t e : waited) tr_wait(s_gather, e);
    CopyArgs a;
    a.src = dev_kv;
    a.src_off = reinterpret_cast<const uint64_t*>(dtab) + g.i0;
    a.src_lstride = dstride;
    a.l_first = g.la;
    a.dst = sp;
    a.chunk = sh.chunk();
    a.nl = g.lb - g.la;
    a.n = g.i1 - g.i0;
    launch(0, a, s_gather, impl_of(cfg, sh.chunk()), 0);
    if (tracing)
      tr("op gather gather r=" + cells(0, dp, dev, n, g.la, g.lb, g.i0, g.i1) + " w=" + ring_cells("SO", roff, seg_bytes));
    CUDA_TRY(cudaEventRecord(full, s_gather));
    tr_record(s_gather, full);

    CUDA_TRY(cudaStreamWaitEvent(s_d2h, full, 0));
    tr_wait(s_d2h, full);
    if (g.i0 == 0) wait_deps(s_d2h, wdeps, g.la, g.lb);  // rule ❸
    if (x->npiece > 1) {
      for (auto& pc : pieces_of(g, sh.chunk(), piece_bytes, runs)) {
        const Seg sub{g.la, g.lb, pc.first, pc.second};
        const uint64_t po = uint64_t(pc.first - g.i0) * sh.chunk();
        host_dmas(hp, host_kv, sh, runs, sub, sp + po, true, cudaMemcpyDeviceToHost, s_d2h);
        if (tracing)
          tr("op d2h d2h r=" + ring_cells("SO", roff + po, uint64_t(pc.second - pc.first) * sh.chunk()) +
             " w=" + cells(1, hp, host, n, g.la, g.lb, pc.first, pc.second));
        cudaEvent_t pe = x->pev[size_t(g.la) * size_t(x->npiece) + size_t(pidx++)];
        CUDA_TRY(cudaEventRecord(pe, s_d2h));
        tr_record(s_d2h, pe);
      }
    } else {
      host_dmas(hp, host_kv, sh, runs, g, sp, true, cudaMemcpyDeviceToHost, s_d2h);
      if (tracing)
        tr("op d2h d2h r=" + ring_cells("SO", roff, seg_bytes) + " w=" + cells(1, hp, host, n, g.la, g.lb, g.i0, g.i1));
    }
    CUDA_TRY(cudaEventRecord(freed, s_d2h));
    tr_record(s_d2h, freed);
    if (g.i1 == n)
      for (int32_t l = g.la; l < g.lb; ++l) record(x, l, s_d2h);
  }
  pc.lap(4);
  if (n == 0)
    for (int32_t l = 0; l < sh.L; ++l) record(x, l, s_d2h);
  record(x, -1, s_d2h);
  pc.lap(5);
  for (int32_t i = 0; i < n; ++i) dp.note_read(dev[i], x->id);
  for (int32_t i = 0; i < n; ++i) hp.note_write(host[i], x->id);
  pc.lap(6);
  if (flags & AEG_FREE_SRC) dp.free(dev, n);
  pc.lap(7);
  return x->id;
}

// ------------------------------------------------------------------------------ swap-in H4
// A writer whose D2H pieces a swap-in can wait on (its own swap-out, or a peer's imported one).
static bool piecewise(const Xfer* w, int32_t L) {
  return w && (w->kind == X_SWAP_OUT || w->kind == X_IMPORTED) && w->npiece > 1 && w->L == L && !w->failed &&
         !w->complete.load();
}

uint64_t Ctx::swap_in(const Shape& sh, const aeg_block* host, const aeg_block* dev, int32_t n, uint32_t flags) {
  return swap_in_from(sh, -1, host, dev, n, 0, flags);
}

uint64_t Ctx::swap_in_from(const Shape& sh, int32_t peer, const aeg_block* host, const aeg_block* dev, int32_t n,
                           uint64_t after, uint32_t flags) {
  AEG_REQUIRE(!host_only, AEG_ERR_STATE, "host-only context has no data path");
  SlabPool& dp = pool[AEG_POOL_DEVICE];
  const bool own = peer < 0;
  SlabPool* hpp = &pool[AEG_POOL_HOST];
  char* hbase = host_kv;
  if (own) {
    hpp->check_owned(host, n, &sh);
  } else {
    auto it = peers.find(peer);
    AEG_REQUIRE(it != peers.end() && it->second->has_host, AEG_ERR_INVALID,
                "peer %d has no imported shared host region", peer);
    AEG_REQUIRE(!(flags & AEG_FREE_SRC), AEG_ERR_INVALID, "AEG_FREE_SRC: a peer's host blocks belong to the peer");
    hpp = &it->second->host_geom;
    hbase = it->second->host_kv;
    hpp->check_geometry(host, n, sh);
    for (int32_t i = 0; i < n; ++i)
      AEG_REQUIRE(block_pool(host[i]) == AEG_POOL_HOST, AEG_ERR_INVALID, "peer handle is not a host block");
  }
  SlabPool& hp = *hpp;
  dp.check_owned(dev, n, &sh);
  AEG_REQUIRE(sh.chunk() <= ring_in.slot_bytes, AEG_ERR_INVALID, "chunk larger than a staging slot");
  if (after) {
    auto it = xfers.find(after);
    AEG_REQUIRE(it == xfers.end() || it->second->L == sh.L || it->second->done_recorded, AEG_ERR_INVALID,
                "dependency transfer %llu has another layer count", (unsigned long long)after);
  }
  Xfer* x = new_xfer(X_SWAP_IN, sh.L, ipc_events(flags) || !own);
  std::vector<uint64_t> rdeps, wdeps;
  if (!(flags & AEG_NO_DEPS)) {
    if (own)
      for (int32_t i = 0; i < n; ++i) hp.deps_for_read(host[i], rdeps);
    for (int32_t i = 0; i < n; ++i) dp.deps_for_write(dev[i], wdeps);
  }
  rdeps = uniq(rdeps);
  wdeps = uniq(wdeps);
  // Rule ❷ at sub-layer granularity: host blocks last written by an in-flight swap-out of this
  // context with D2H pieces are waited for per piece (the highest piece of that swap-out holding
  // any block of our piece; its pieces land in order on one stream).  Other writers (and the
  // cross-instance `after`): per-layer events.
  std::vector<Xfer*> pdeps;
  {
    std::vector<uint64_t> rest;
    for (uint64_t d : rdeps) {
      auto it = xfers.find(d);
      Xfer* w = it == xfers.end() ? nullptr : it->second.get();
      if (piecewise(w, sh.L))
        pdeps.push_back(w);
      else
        rest.push_back(d);
    }
    rdeps.swap(rest);
  }
  Xfer* after_x = nullptr;  // `after` waited per piece: a piece none of whose blocks it wrote still
                            // waits for its layer to land (aeg.h: layer l waits on layer l of after)
  if (after) {  // rule ❷ across instances (Fig. 10 ③): per piece if the peer exported pieces
    auto it = xfers.find(after);
    if (it != xfers.end() && piecewise(it->second.get(), sh.L)) {
      after_x = it->second.get();
      if (std::find(pdeps.begin(), pdeps.end(), after_x) == pdeps.end()) pdeps.push_back(after_x);
    } else
      rdeps.push_back(after);
  }
  rdeps = uniq(rdeps);
  char *htab = nullptr, *dtab = nullptr;
  if (n > 0) {
    alloc_table(uint64_t(n) * 8, x->id, &htab, &dtab);
    uint64_t* t = reinterpret_cast<uint64_t*>(htab);
    for (int32_t i = 0; i < n; ++i) t[i] = dp.off0(dev[i], sh);
    // fetched on the scatter stream by a kernel (no copy-engine op on a kernel stream: with CUDA
    // timing events around the scatters one made every scatter wait for the H2D stream to block on
    // a ring slot, profiles/r01/timeline.txt; and no H2D copy queued behind other transfers' DMAs)
    fetch_table(dtab, htab, uint64_t(n) * 8, s_scatter);
  }
  const auto segs = plan(sh.L, n, sh.chunk(), ring_in.slot_bytes, uint64_t(cfg.pack_layer_mib) << 20);
  const auto runs = runs_of(host, n);
  const uint64_t dstride = dp.lstride(sh);
  const uint64_t piece_bytes = uint64_t(cfg.dma_piece_mib) << 20;
  // per piece of a layer (same block ranges in every layer): (writer, its highest piece) to wait on
  std::vector<std::vector<std::pair<Xfer*, int32_t>>> pneed;
  if (!pdeps.empty()) {
    for (const Seg& g : segs) {
      if (g.la != 0) break;
      for (auto& pc : pieces_of(g, sh.chunk(), piece_bytes, runs)) {
        std::vector<std::pair<Xfer*, int32_t>> need;
        for (Xfer* w : pdeps) {
          int32_t hi = -1;
          for (int32_t i = pc.first; i < pc.second; ++i) {
            auto f = w->wpos.find(host[i]);
            if (f == w->wpos.end()) continue;
            const int32_t p = int32_t(std::upper_bound(w->piece_lo.begin(), w->piece_lo.end(), f->second) -
                                      w->piece_lo.begin()) - 1;
            hi = std::max(hi, p);
          }
          if (hi < 0 && w == after_x) hi = w->npiece - 1;  // its last piece of the layer = the layer
          if (hi >= 0) need.push_back({w, hi});
        }
        pneed.push_back(std::move(need));
      }
    }
  }
  int32_t pidx = 0;
  for (const Seg& g : segs) {
    if (g.i0 == 0) pidx = 0;
    if (g.i0 == 0) wait_deps(s_h2d, rdeps, g.la, g.lb);  // rule ❷ per layer (reading 12)
    cudaEvent_t full, freed;
    uint64_t roff;
    std::vector<cudaEvent_t> waited;
    const uint64_t seg_bytes = uint64_t(g.lb - g.la) * uint64_t(g.i1 - g.i0) * sh.chunk();
    char* sp = ring_in.acquire(seg_bytes, s_h2d, &full, &freed, &roff, tracing ? &waited : nullptr);
    for (cudaEvent_t e : waited) tr_wait(s_h2d, e);
    if (!pneed.empty()) {
      for (auto& pc : pieces_of(g, sh.chunk(), piece_bytes, runs)) {
        for (auto& nd : pneed[size_t(pidx)])
          for (int32_t l = g.la; l < g.lb; ++l) {
            cudaEvent_t e = nd.first->pev[size_t(l) * size_t(nd.first->npiece) + size_t(nd.second)];
            CUDA_TRY(cudaStreamWaitEvent(s_h2d, e, 0));
            tr_wait(s_h2d, e);
          }
        ++pidx;
        const Seg sub{g.la, g.lb, pc.first, pc.second};
        const uint64_t po = uint64_t(pc.first - g.i0) * sh.chunk();
        host_dmas(hp, hbase, sh, runs, sub, sp + po, false, cudaMemcpyHostToDevice, s_h2d);
        if (tracing)
          tr("op h2d h2d r=" + cells(1, hp, host, n, g.la, g.lb, pc.first, pc.second) + " w=" +
             ring_cells("SI", roff + po, uint64_t(pc.second - pc.first) * sh.chunk()));
      }
    } else {
      host_dmas(hp, hbase, sh, runs, g, sp, false, cudaMemcpyHostToDevice, s_h2d);
      if (tracing)
        tr("op h2d h2d r=" + cells(1, hp, host, n, g.la, g.lb, g.i0, g.i1) + " w=" + ring_cells("SI", roff, seg_bytes));
    }
    CUDA_TRY(cudaEventRecord(full, s_h2d));
    tr_record(s_h2d, full);

    CUDA_TRY(cudaStreamWaitEvent(s_scatter, full, 0));
    tr_wait(s_scatter, full);
    if (g.i0 == 0) wait_deps(s_scatter, wdeps, g.la, g.lb);  // rule ❸
    CopyArgs a;
    a.src = sp;
    a.dst = dev_kv;
    a.dst_off = reinterpret_cast<const uint64_t*>(dtab) + g.i0;
    a.dst_lstride = dstride;
    a.l_first = g.la;
    a.chunk = sh.chunk();
    a.nl = g.lb - g.la;
    a.n = g.i1 - g.i0;
    launch(1, a, s_scatter, impl_of(cfg, sh.chunk()), 0);
    if (tracing)
      tr("op scatter scatter r=" + ring_cells("SI", roff, seg_bytes) + " w=" + cells(0, dp, dev, n, g.la, g.lb, g.i0, g.i1));
    CUDA_TRY(cudaEventRecord(freed, s_scatter));
    tr_record(s_scatter, freed);
    if (g.i1 == n)
      for (int32_t l = g.la; l < g.lb; ++l) record(x, l, s_scatter);
  }
  if (n == 0)
    for (int32_t l = 0; l < sh.L; ++l) record(x, l, s_scatter);
  record(x, -1, s_scatter);
  if (own)
    for (int32_t i = 0; i < n; ++i) hp.note_read(host[i], x->id);
  for (int32_t i = 0; i < n; ++i) dp.note_write(dev[i], x->id);
  if (own && (flags & AEG_FREE_SRC)) hp.free(host, n);
  return x->id;
}

// ------------------------------------------------------------------------------- migrate H5
uint64_t Ctx::migrate(const Shape& sh, const aeg_block* src, int32_t peer, const aeg_block* dst, int32_t n,
                      uint32_t flags) {
  AEG_REQUIRE(!host_only, AEG_ERR_STATE, "host-only context has no data path");
  SlabPool& dp = pool[AEG_POOL_DEVICE];
  dp.check_owned(src, n, &sh);
  const SlabPool* dg = &dp;
  char* dbase = dev_kv;
  Peer* P = nullptr;
  if (peer < 0) {
    dp.check_owned(dst, n, &sh);
    std::vector<aeg_block> all(src, src + n);
    all.insert(all.end(), dst, dst + n);
    std::sort(all.begin(), all.end());
    AEG_REQUIRE(std::adjacent_find(all.begin(), all.end()) == all.end(), AEG_ERR_INVALID,
                "local migrate: source and destination blocks overlap");
  } else {
    auto it = peers.find(peer);
    AEG_REQUIRE(it != peers.end() && it->second->valid, AEG_ERR_INVALID, "peer %d not imported", peer);
    P = it->second.get();
    P->geom.check_geometry(dst, n, sh);
    dg = &P->geom;
    dbase = P->dev_kv;
  }
  AEG_REQUIRE(!(flags & AEG_MIGRATE_CE) || sh.chunk() <= ring_out.slot_bytes, AEG_ERR_INVALID,
              "copy-engine route: chunk larger than a staging slot");
  Xfer* x = new_xfer(X_MIGRATE, sh.L, ipc_events(flags) || (peer >= 0 && !P->same_process));
  std::vector<uint64_t> rdeps, wdeps;
  if (!(flags & AEG_NO_DEPS)) {
    for (int32_t i = 0; i < n; ++i) dp.deps_for_read(src[i], rdeps);
    if (peer < 0)
      for (int32_t i = 0; i < n; ++i) dp.deps_for_write(dst[i], wdeps);
  }
  rdeps = uniq(rdeps);
  wdeps = uniq(wdeps);
  for (uint64_t d : wdeps) rdeps.push_back(d);
  rdeps = uniq(rdeps);
  char *htab = nullptr, *dtab = nullptr;
  if (n > 0 && !(flags & AEG_MIGRATE_CE)) {
    alloc_table(uint64_t(n) * 16, x->id, &htab, &dtab);
    uint64_t* t = reinterpret_cast<uint64_t*>(htab);
    for (int32_t i = 0; i < n; ++i) t[i] = dp.off0(src[i], sh);
    for (int32_t i = 0; i < n; ++i) t[n + i] = dg->off0(dst[i], sh);
    fetch_table(dtab, htab, uint64_t(n) * 16, s_migrate);
  }
  if (flags & AEG_MIGRATE_CE) {
    // Copy-engine route (SURVEY H5 alternative; zero SMs on the link): per segment of the out
    // staging ring, the gather kernel packs the source blocks (HBM), then copy engines move the
    // segment into the destination pool — one command per destination run and layer, or one 2-D
    // command per layer across equal whole runs (host_dmas) — on s_p2p; per-layer events there.
    if (n > 0) {
      alloc_table(uint64_t(n) * 8, x->id, &htab, &dtab);
      uint64_t* t = reinterpret_cast<uint64_t*>(htab);
      for (int32_t i = 0; i < n; ++i) t[i] = dp.off0(src[i], sh);
      fetch_table(dtab, htab, uint64_t(n) * 8, s_gather);
    }
    const auto segs = plan(sh.L, n, sh.chunk(), ring_out.slot_bytes, uint64_t(cfg.pack_layer_mib) << 20);
    const auto runs = runs_of(dst, n);
    const uint64_t sstride = dp.lstride(sh);
    for (const Seg& g : segs) {
      if (g.i0 == 0) wait_deps(s_gather, rdeps, g.la, g.lb);  // rules ❷ (sources) and ❸ (local dst)
      cudaEvent_t full, freed;
      uint64_t roff;
      std::vector<cudaEvent_t> waited;
      const uint64_t seg_bytes = uint64_t(g.lb - g.la) * uint64_t(g.i1 - g.i0) * sh.chunk();
      char* sp = ring_out.acquire(seg_bytes, s_gather, &full, &freed, &roff, tracing ? &waited : nullptr);
      for (cudaEvent_t e : waited) tr_wait(s_gather, e);
      CopyArgs a;
      a.src = dev_kv;
      a.src_off = reinterpret_cast<const uint64_t*>(dtab) + g.i0;
      a.src_lstride = sstride;
      a.l_first = g.la;
      a.dst = sp;
      a.chunk = sh.chunk();
      a.nl = g.lb - g.la;
      a.n = g.i1 - g.i0;
      launch(0, a, s_gather, impl_of(cfg, sh.chunk()), 0);
      if (tracing)
        tr("op gather gather r=" + cells(0, dp, src, n, g.la, g.lb, g.i0, g.i1) + " w=" + ring_cells("SO", roff, seg_bytes));
      CUDA_TRY(cudaEventRecord(full, s_gather));
      tr_record(s_gather, full);
      CUDA_TRY(cudaStreamWaitEvent(s_p2p, full, 0));
      tr_wait(s_p2p, full);
      host_dmas(*dg, dbase, sh, runs, g, sp, true, cudaMemcpyDefault, s_p2p);
      if (tracing)
        tr("op p2p p2p r=" + ring_cells("SO", roff, seg_bytes) + " w=" +
           cells(peer < 0 ? 0 : 2, *dg, dst, n, g.la, g.lb, g.i0, g.i1));
      CUDA_TRY(cudaEventRecord(freed, s_p2p));
      tr_record(s_p2p, freed);
      if (g.i1 == n)
        for (int32_t l = g.la; l < g.lb; ++l) record(x, l, s_p2p);
    }
    if (n == 0)
      for (int32_t l = 0; l < sh.L; ++l) record(x, l, s_p2p);
    record(x, -1, s_p2p);
    for (int32_t i = 0; i < n; ++i) dp.note_read(src[i], x->id);
    if (peer < 0)
      for (int32_t i = 0; i < n; ++i) dp.note_write(dst[i], x->id);
    if (flags & AEG_FREE_SRC) dp.free(src, n);
    return x->id;
  }
  // Layers per launch.  A launch boundary costs a fixed ~15 us (ramp + drain of the streaming
  // pipeline; not hidden by a second kernel stream, whose concurrent CTAs lose as much to DRAM
  // efficiency): one configs[2] hand-off (16 Llama-2-13B requests, 733 MiB per layer) takes 10.09 ms
  // as 40 launches, 9.70 ms as 8 and 9.48 ms as 1 (profiles/r02/migrate_pack.txt).  So pack layers up
  // to >= ~1 ms of copying per launch: 4 GiB on the same GPU (HBM speed), 512 MiB over NVLink
  // (~0.7 ms at the measured 770 GB/s peer copy).  Every layer still gets its event, recorded when
  // its launch completes; layers larger than the pack go one per launch.
  const bool remote = P && (!P->same_process || P->device != device);
  const uint64_t pack = remote ? (512ull << 20) : (uint64_t(AEG_MIGRATE_LOCAL_PACK_MIB) << 20);
  const uint64_t layer = uint64_t(n) * sh.chunk();
  int32_t lps = 1;
  if (n > 0 && layer < pack) lps = int32_t(std::min<uint64_t>(sh.L, std::max<uint64_t>(1, pack / layer)));
  // Paged -> paged under AUTO (WARP for tiny chunks).  Remote: LSU, plain st.global to the peer
  // aperture (bulk copies into another GPU's memory are not relied on).  Local: BULKW — with both
  // sides paged over tens of GB the single-issuer BULK ring loses to LSU, the 4-issuer BULKW beats
  // both (profiles/r02/migrate_leg_probe_r02.txt, 16 Llama-2-13B requests, 30 GB per side, the four
  // layout pairs: BULKW 5.54-5.96 TB/s, LSU 5.36-5.82, BULK 5.02-5.22; 4 requests: BULKW 5.44-5.61,
  // BULK 5.38-5.66, LSU 5.34-5.53).
  const int impl = cfg.kernel != AEG_KERNEL_AUTO ? impl_of(cfg, sh.chunk())
                   : sh.chunk() <= (4u << 10)    ? IMPL_WARP
                   : remote                      ? IMPL_LSU
                                                 : IMPL_BULKW;
  for (int32_t la = 0; la < sh.L; la += lps) {
    const int32_t lb = std::min(sh.L, la + lps);
    if (n > 0) {
      wait_deps(s_migrate, rdeps, la, lb);
      CopyArgs a;
      a.src = dev_kv;
      a.src_off = reinterpret_cast<const uint64_t*>(dtab);
      a.src_lstride = dp.lstride(sh);
      a.dst = dbase;
      a.dst_off = reinterpret_cast<const uint64_t*>(dtab) + n;
      a.dst_lstride = dg->lstride(sh);
      a.l_first = la;
      a.chunk = sh.chunk();
      a.nl = lb - la;
      a.n = n;
      launch(2, a, s_migrate, impl, cfg.migrate_ctas);
      if (tracing)
        tr("op migrate migrate r=" + cells(0, dp, src, n, la, lb, 0, n) + " w=" + cells(peer < 0 ? 0 : 2, *dg, dst, n, la, lb, 0, n));
    }
    for (int32_t l = la; l < lb; ++l) record(x, l, s_migrate);
  }
  record(x, -1, s_migrate);
  for (int32_t i = 0; i < n; ++i) dp.note_read(src[i], x->id);
  if (peer < 0)
    for (int32_t i = 0; i < n; ++i) dp.note_write(dst[i], x->id);
  if (flags & AEG_FREE_SRC) dp.free(src, n);
  return x->id;
}

// ------------------------------------------------------------------------------ relocate N1
uint64_t Ctx::relocate(uint64_t src_off, uint64_t dst_off, uint64_t bytes) {
  AEG_REQUIRE(!host_only, AEG_ERR_STATE, "host-only context has no data path");
  const uint64_t W = cfg.device_weight_bytes;
  AEG_REQUIRE(src_off + bytes <= W && dst_off + bytes <= W, AEG_ERR_INVALID, "relocation outside the weights region");
  AEG_REQUIRE(src_off % 16 == 0 && dst_off % 16 == 0 && bytes % 16 == 0, AEG_ERR_INVALID,
              "relocation offsets and size must be multiples of 16");
  Xfer* x = new_xfer(X_RELOCATE, 1, false);
  int nl = 0;
  // Not bracketed by CUDA timing events even under AEG_CFG_TIMING: the weights stream also carries
  // copy-engine DMAs, and timing events on a stream that mixes copy-engine ops and kernels held the
  // kernel until other streams' queued H2D drained — a switch's relocation would
  // wait for the incoming KV.  Its launches and bytes are still counted.
  cudaError_t e = launch_memmove(dev_w, src_off, dst_off, bytes, impl_of(cfg, bytes), s_weights, &nl);
  AEG_REQUIRE(e == cudaSuccess, AEG_ERR_CUDA, "relocate launch failed: %s", cudaGetErrorString(e));
  kstats[3].launches += nl;
  kstats[3].bytes += 2 * bytes;
  record(x, 0, s_weights);
  record(x, -1, s_weights);
  return x->id;
}

}  // namespace aeg
