// Weight staging (H7): Model Cache -> pinned Stage Buffer ring -> copy-engine H2D into the bump-
// allocated weights region, "in a multi-threaded, chunked, and pipelined manner".
//
// Pipeline per job (one aeg_weights_stage call):
//   * the device range [start, end) of the job's shards is cut into stage_chunk_bytes chunks;
//   * T worker threads fill chunk images in pinned Stage Buffer slots (shard extraction for
//     Megatron COL/ROW/VOCAB splits happens here; padding between shards is zeroed); a worker
//     first waits for the slot's previous DMA (cudaEventSynchronize on the slot event);
//   * one issuer thread issues, in chunk order, one cudaMemcpyAsync H2D per chunk on s_weights,
//     records the slot event and every layer event whose last byte is in the chunk.
// When every tensor lies in host memory registered with aeg_host_register the workers are skipped
// and the issuer DMAs shards straight from the Model Cache (2-D copies for ROW shards).
#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <functional>

#if defined(__x86_64__)
#include <emmintrin.h>
#endif

#include "engine.h"

namespace aeg {

namespace {

// Fill copy into the pinned Stage Buffer with streaming (non-temporal) stores.  A regular store
// first reads the destination line (read-for-ownership), so memcpy costs the staged path 4 host-
// DRAM passes per byte (Model Cache read, slot RFO, slot write, DMA read) and glibc only streams
// above a threshold larger than one fill part.  Measured with a copy engine streaming H2D from the
// same buffer (tools/ntcopy_probe.cc, profiles/r01/ntcopy_probe.txt): memcpy 42 GB/s vs streaming
// 59-65 GB/s of fill.  The caller fences (stream_fence) before the chunk is handed to the issuer.
void stream_copy(char* dst, const char* src, uint64_t n) {
#if defined(__x86_64__)
  uint64_t i = 0;
  const uint64_t head = (64 - (reinterpret_cast<uintptr_t>(dst) & 63)) & 63;
  if (head) {
    const uint64_t h = head < n ? head : n;
    std::memcpy(dst, src, h);
    i = h;
  }
  for (; i + 64 <= n; i += 64) {
    const __m128i a = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i));
    const __m128i b = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 16));
    const __m128i c = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 32));
    const __m128i d = _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i + 48));
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i), a);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 16), b);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 32), c);
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i + 48), d);
  }
  if (i < n) std::memcpy(dst + i, src + i, n - i);
#else
  std::memcpy(dst, src, n);
#endif
}

// Make the streaming stores globally visible before the filled part is published (they are weakly
// ordered; the mutex that publishes it does not order them).
void stream_fence() {
#if defined(__x86_64__)
  _mm_sfence();
#endif
}

uint64_t shard_bytes(const aeg_weight_desc& d, int32_t tp) {
  const uint64_t all = d.rows * d.cols * uint64_t(d.elem_bytes);
  return d.split == AEG_SPLIT_REPLICATED ? all : all / uint64_t(tp);
}

// Copy bytes [a, b) of rank r's shard of tensor d into dst (Megatron splits, reading 18).  The copy
// granularity of contiguous ranges was swept (16 KiB .. one memcpy per range): no measurable effect
// on the staged switch (profiles/r01/sweep3).
void copy_shard(char* dst, const aeg_weight_desc& d, int32_t r, int32_t tp, uint64_t a, uint64_t b) {
  const char* src = static_cast<const char*>(d.host_src);
  const uint64_t row = d.cols * uint64_t(d.elem_bytes);
  if (d.split == AEG_SPLIT_REPLICATED || tp == 1) {  // the shard is the whole, contiguous tensor
    stream_copy(dst, src + a, b - a);
    return;
  }
  if (d.split == AEG_SPLIT_COL || d.split == AEG_SPLIT_VOCAB) {
    const uint64_t g_rows = d.rows / uint64_t(d.groups);
    const uint64_t part_rows = g_rows / uint64_t(tp);
    const uint64_t part = part_rows * row;  // contiguous bytes of one group's part
    for (uint64_t x = a; x < b;) {
      const uint64_t gi = x / part, in = x - gi * part;
      const uint64_t len = std::min(b - x, part - in);
      stream_copy(dst + (x - a), src + (gi * g_rows + uint64_t(r) * part_rows) * row + in, len);
      x += len;
    }
    return;
  }
  // ROW: every row contributes the column range [r*cols/tp, (r+1)*cols/tp)
  const uint64_t w = row / uint64_t(tp);
  for (uint64_t x = a; x < b;) {
    const uint64_t rho = x / w, in = x - rho * w;
    const uint64_t len = std::min(b - x, w - in);
    stream_copy(dst + (x - a), src + rho * row + uint64_t(r) * w + in, len);
    x += len;
  }
}

}  // namespace

struct WJob {
  Xfer* x = nullptr;
  std::vector<aeg_weight_desc> d;
  std::vector<uint64_t> off, size;
  int32_t r = 0, tp = 1;
  uint64_t start = 0, end = 0;
  bool direct = false;
};

struct WeightPipe {
  Ctx* c = nullptr;
  std::thread issuer;
  std::vector<std::thread> workers;
  std::mutex m;
  std::condition_variable cv_job, cv_task, cv_filled;
  std::deque<std::unique_ptr<WJob>> jobs;
  std::deque<std::function<void()>> tasks;
  std::vector<uint8_t> filled;  // per chunk of the current job: parts filled so far
  int64_t outstanding = 0;      // fill tasks queued or running (they point into the current job)
  static constexpr int kParts = 8;  // fill tasks per chunk (8 MiB each for 64 MiB chunks)
  bool stop = false;
  int nslots = 0;
  uint64_t chunk = 0;
  uint64_t next_slot = 0;
  std::vector<cudaEvent_t> slot_ev;
  std::vector<uint8_t> slot_used;
  // counters (aeg_weights_stats)
  std::atomic<uint64_t> n_chunks{0};
  std::atomic<uint64_t> wait_fill_ns{0}, wait_slot_ns{0};

  static uint64_t now_ns() {
    return uint64_t(std::chrono::duration_cast<std::chrono::nanoseconds>(
                        std::chrono::steady_clock::now().time_since_epoch())
                        .count());
  }

  void worker_loop() {
    cudaSetDevice(c->device);
    for (;;) {
      std::function<void()> t;
      {
        std::unique_lock<std::mutex> lk(m);
        cv_task.wait(lk, [&] { return stop || !tasks.empty(); });
        if (tasks.empty()) return;
        t = std::move(tasks.front());
        tasks.pop_front();
      }
      t();
    }
  }

  // Fill the Stage Buffer slot with the device image of [cs, ce) of job j.
  // Fill part `part` of `parts` of chunk ci (the parts of one chunk are queued back to back, so all
  // threads finish chunk 0 first and its DMA starts after ~1 ms instead of after a whole-chunk copy).
  void fill(WJob* j, uint64_t ci, int slot, bool wait_slot, int part, int parts) {
    if (wait_slot) {  // rule ❸ for the Stage Buffer slot
      const uint64_t t0 = now_ns();
      cudaEventSynchronize(slot_ev[slot]);
      wait_slot_ns += now_ns() - t0;
    }
    const uint64_t c0 = j->start + ci * chunk, c1 = std::min(j->end, c0 + chunk);
    const uint64_t span = (c1 - c0 + parts - 1) / parts;
    const uint64_t cs = std::min(c1, c0 + span * part), ce = std::min(c1, cs + span);
    char* dst = c->host_stage + uint64_t(slot) * chunk + (cs - c0);
    uint64_t p = cs;
    auto k0 = std::upper_bound(j->off.begin(), j->off.end(), cs) - j->off.begin();
    for (size_t k = k0 > 0 ? k0 - 1 : 0; k < j->d.size() && j->off[k] < ce; ++k) {
      const uint64_t ts = j->off[k], te = ts + j->size[k];
      if (te <= cs) continue;
      const uint64_t a = std::max(ts, cs), b = std::min(te, ce);
      if (a > p) std::memset(dst + (p - cs), 0, a - p);
      copy_shard(dst + (a - cs), j->d[k], j->r, j->tp, a - ts, b - ts);
      p = b;
    }
    if (ce > p) std::memset(dst + (p - cs), 0, ce - p);
    stream_fence();
    bool wake;
    {
      std::lock_guard<std::mutex> lk(m);
      wake = ++filled[ci] == parts;
      wake = (--outstanding == 0) || wake;
    }
    if (wake) cv_filled.notify_all();
  }

  void record_layers(WJob* j, const std::vector<uint64_t>& layer_last, uint64_t upto, cudaStream_t s) {
    {
      std::lock_guard<std::mutex> g(c->mu);
      for (int32_t l = 0; l < j->x->L; ++l)
        if (!j->x->recorded[l] && layer_last[l] != ~0ull && layer_last[l] < upto) c->record(j->x, l, s);
    }
    c->cv.notify_all();  // wake WAIT_STREAM / BLOCK readiness waiters (aeg_layer_ready)
  }

  void run_job(WJob* j) {
    cudaStream_t s = c->s_weights;
    // last device byte (+1) of every readiness layer
    std::vector<uint64_t> layer_last(j->x->L, ~0ull);
    for (size_t k = 0; k < j->d.size(); ++k) {
      uint64_t& v = layer_last[j->d[k].layer];
      const uint64_t e = j->off[k] + j->size[k];
      v = (v == ~0ull) ? e : std::max(v, e);
    }
    for (auto& v : layer_last)
      if (v != ~0ull) v -= 1;  // index of the last byte
    try {
      if (j->direct) {
        // Pace the issue: at most kWindow chunks of DMA queued on s_weights, so copies other
        // streams enqueue meanwhile (the switch's KV swap-in) are not stuck behind the whole model.
        constexpr int kWindow = 4;
        uint64_t since = 0, marks = 0;
        for (size_t k = 0; k < j->d.size(); ++k) {
          if (since >= chunk) {
            const int slot = int(marks++ % uint64_t(kWindow));
            if (marks > uint64_t(kWindow)) CUDA_TRY(cudaEventSynchronize(slot_ev[slot]));
            CUDA_TRY(cudaEventRecord(slot_ev[slot], s));
            since = 0;
          }
          since += j->size[k];
          const aeg_weight_desc& d = j->d[k];
          char* dst = c->dev_w + j->off[k];
          const char* src = static_cast<const char*>(d.host_src);
          const uint64_t row = d.cols * uint64_t(d.elem_bytes);
          if (d.split == AEG_SPLIT_REPLICATED || j->tp == 1) {
            CUDA_TRY(cudaMemcpyAsync(dst, src, j->size[k], cudaMemcpyHostToDevice, s));
          } else if (d.split == AEG_SPLIT_ROW) {
            const uint64_t w = row / uint64_t(j->tp);
            CUDA_TRY(cudaMemcpy2DAsync(dst, w, src + uint64_t(j->r) * w, row, w, d.rows, cudaMemcpyHostToDevice, s));
          } else {
            const uint64_t g_rows = d.rows / uint64_t(d.groups), part_rows = g_rows / uint64_t(j->tp);
            for (int32_t gi = 0; gi < d.groups; ++gi)
              CUDA_TRY(cudaMemcpyAsync(dst + uint64_t(gi) * part_rows * row,
                                       src + (uint64_t(gi) * g_rows + uint64_t(j->r) * part_rows) * row,
                                       part_rows * row, cudaMemcpyHostToDevice, s));
          }
          const uint64_t te = j->off[k] + j->size[k];
          const uint64_t next = k + 1 < j->d.size() ? j->off[k + 1] : std::min(j->end, align_up(te, 256));
          if (next > te) CUDA_TRY(cudaMemsetAsync(c->dev_w + te, 0, next - te, s));
          record_layers(j, layer_last, te, s);
        }
      } else {
        const uint64_t nch = (j->end - j->start + chunk - 1) / chunk;
        std::vector<int> slot_of(nch);
        {
          std::lock_guard<std::mutex> lk(m);
          filled.assign(nch, 0);
        }
        uint64_t dispatched = 0;
        for (uint64_t ci = 0; ci < nch; ++ci) {
          // keep up to nslots chunks in flight (slots of chunks < ci are already issued)
          while (dispatched < nch && dispatched < ci + uint64_t(nslots)) {
            const int slot = int(next_slot++ % uint64_t(nslots));
            slot_of[dispatched] = slot;
            const bool w = slot_used[slot] != 0;
            const uint64_t q = dispatched;
            {
              std::lock_guard<std::mutex> lk(m);
              for (int part = 0; part < kParts; ++part)
                tasks.push_back([this, j, q, slot, w, part] { fill(j, q, slot, w, part, kParts); });
              outstanding += kParts;
            }
            cv_task.notify_all();
            ++dispatched;
          }
          {
            const uint64_t t0 = now_ns();
            std::unique_lock<std::mutex> lk(m);
            cv_filled.wait(lk, [&] { return filled[ci] == kParts; });
            wait_fill_ns += now_ns() - t0;
          }
          n_chunks++;
          const uint64_t cs = j->start + ci * chunk, ce = std::min(j->end, cs + chunk);
          const int slot = slot_of[ci];
          CUDA_TRY(cudaMemcpyAsync(c->dev_w + cs, c->host_stage + uint64_t(slot) * chunk, ce - cs,
                                   cudaMemcpyHostToDevice, s));
          CUDA_TRY(cudaEventRecord(slot_ev[slot], s));
          slot_used[slot] = 1;
          record_layers(j, layer_last, ce, s);
        }
      }
      std::lock_guard<std::mutex> g(c->mu);
      for (int32_t l = 0; l < j->x->L; ++l)
        if (!j->x->recorded[l]) c->record(j->x, l, s);  // layers without tensors
      c->record(j->x, -1, s);
      c->w_inflight--;
    } catch (const std::exception& e) {  // aeg::Error (CUDA failures) or host allocation failure
      fprintf(stderr, "aegkv: weight pipeline failed: %s\n", e.what());
      {  // fill tasks already dispatched point into this job: let them finish before it is freed
        std::unique_lock<std::mutex> lk(m);
        cv_filled.wait(lk, [&] { return outstanding == 0; });
      }
      cudaStreamSynchronize(s);
      (void)cudaGetLastError();
      std::lock_guard<std::mutex> g(c->mu);
      std::fill(j->x->recorded.begin(), j->x->recorded.end(), uint8_t(1));  // never block a waiter
      j->x->done_recorded = true;
      j->x->failed = true;
      j->x->complete.store(true);
      c->w_inflight--;
    }
    c->cv.notify_all();
  }

  void issuer_loop() {
    cudaSetDevice(c->device);
    for (;;) {
      std::unique_ptr<WJob> j;
      {
        std::unique_lock<std::mutex> lk(m);
        cv_job.wait(lk, [&] { return stop || !jobs.empty(); });
        if (jobs.empty()) return;
        j = std::move(jobs.front());
        jobs.pop_front();
      }
      run_job(j.get());
    }
  }
};

Ctx::Ctx() = default;
Ctx::~Ctx() = default;

void Ctx::weights_counters(uint64_t* chunks, double* wait_fill_ms, double* wait_slot_ms) {
  if (chunks) *chunks = wp ? wp->n_chunks.load() : 0;
  if (wait_fill_ms) *wait_fill_ms = wp ? wp->wait_fill_ns.load() * 1e-6 : 0.0;
  if (wait_slot_ms) *wait_slot_ms = wp ? wp->wait_slot_ns.load() * 1e-6 : 0.0;
}

void Ctx::weights_start() {
  wp = std::make_unique<WeightPipe>();
  wp->c = this;
  wp->chunk = cfg.stage_chunk_bytes;
  wp->nslots = int(cfg.stage_ring_bytes / cfg.stage_chunk_bytes);
  wp->slot_ev.resize(wp->nslots);
  wp->slot_used.assign(wp->nslots, 0);
  for (auto& e : wp->slot_ev) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming | cudaEventBlockingSync));
  wp->issuer = std::thread([p = wp.get()] { p->issuer_loop(); });
  const int T = std::max(1, cfg.host_threads);
  for (int i = 0; i < T; ++i) wp->workers.emplace_back([p = wp.get()] { p->worker_loop(); });
}

void Ctx::weights_stop() {
  if (!wp) return;
  {
    std::lock_guard<std::mutex> lk(wp->m);
    wp->stop = true;
  }
  wp->cv_job.notify_all();
  wp->cv_task.notify_all();
  if (wp->issuer.joinable()) wp->issuer.join();
  for (auto& t : wp->workers) t.join();
  for (auto& e : wp->slot_ev) cudaEventDestroy(e);
  wp.reset();
}

// Validation + bump allocation happen here, under the context mutex.
uint64_t Ctx::weights_stage(const aeg_weight_desc* d, int32_t n, int32_t r, int32_t tp, uint64_t* offs) {
  AEG_REQUIRE(!host_only, AEG_ERR_STATE, "host-only context has no data path");
  AEG_REQUIRE(n >= 0 && (n == 0 || (d && offs)), AEG_ERR_INVALID, "bad descriptor array");
  AEG_REQUIRE(tp >= 1 && r >= 0 && r < tp, AEG_ERR_INVALID, "bad tp rank %d / size %d", r, tp);
  auto j = std::make_unique<WJob>();
  j->d.assign(d, d + n);
  j->r = r;
  j->tp = tp;
  int32_t L = 1;
  uint64_t p = w_bump;
  bool direct = n > 0;
  for (int32_t k = 0; k < n; ++k) {
    const aeg_weight_desc& t = d[k];
    AEG_REQUIRE(t.host_src && t.rows > 0 && t.cols > 0 && t.elem_bytes > 0 && t.layer >= 0 && t.layer < 1 << 20,
                AEG_ERR_INVALID, "tensor %d: bad descriptor", k);
    AEG_REQUIRE(t.split >= AEG_SPLIT_REPLICATED && t.split <= AEG_SPLIT_VOCAB, AEG_ERR_INVALID, "tensor %d: bad split", k);
    AEG_REQUIRE(t.groups >= 1, AEG_ERR_INVALID, "tensor %d: groups must be >= 1", k);
    if (t.split == AEG_SPLIT_COL || t.split == AEG_SPLIT_VOCAB)
      AEG_REQUIRE(t.rows % (uint64_t(t.groups) * tp) == 0, AEG_ERR_INVALID, "tensor %d: rows %llu not divisible by %d",
                  k, (unsigned long long)t.rows, t.groups * tp);
    if (t.split == AEG_SPLIT_ROW)
      AEG_REQUIRE(t.cols % uint64_t(tp) == 0 && t.groups == 1, AEG_ERR_INVALID, "tensor %d: cols not divisible by tp", k);
    const uint64_t sz = shard_bytes(t, tp);
    j->off.push_back(p);
    j->size.push_back(sz);
    p = align_up(p + sz, 256);
    L = std::max(L, t.layer + 1);
    const char* s = static_cast<const char*>(t.host_src);
    const uint64_t all = t.rows * t.cols * uint64_t(t.elem_bytes);
    bool reg = false;
    for (auto& rg : registered)
      if (s >= rg.first && s + all <= rg.first + rg.second) reg = true;
    direct = direct && reg;
  }
  // the region must hold the shards, [start, off_last + size_last) (reading 17, oracle O8); the
  // padding after the last shard is written only up to the region's end
  const uint64_t data_end = n > 0 ? j->off.back() + j->size.back() : w_bump;
  AEG_REQUIRE(data_end <= cfg.device_weight_bytes, AEG_ERR_OOM, "weights region exhausted: need %llu of %llu bytes",
              (unsigned long long)data_end, (unsigned long long)cfg.device_weight_bytes);
  std::copy(j->off.begin(), j->off.end(), offs);
  j->start = w_bump;
  j->end = std::min(p, cfg.device_weight_bytes);  // through the last shard's padding (zeros, reading 17)
  j->direct = direct;
  w_bump = p;
  Xfer* x = new_xfer(X_WEIGHTS, L, false);
  j->x = x;
  w_inflight++;
  {
    std::lock_guard<std::mutex> lk(wp->m);
    wp->jobs.push_back(std::move(j));
  }
  wp->cv_job.notify_one();
  return x->id;
}

}  // namespace aeg
