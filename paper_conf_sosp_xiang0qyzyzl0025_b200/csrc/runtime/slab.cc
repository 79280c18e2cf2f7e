#include "slab.h"

#include <algorithm>

namespace aeg {

void SlabPool::init(int pool_id, uint64_t bytes, uint64_t sbytes, int lay) {
  AEG_REQUIRE(sbytes > 0 && sbytes % 16 == 0, AEG_ERR_INVALID,
              "slab size must be a positive multiple of 16 bytes (16-byte vector and bulk copies)");
  AEG_REQUIRE(lay == AEG_LAYER_MAJOR || lay == AEG_BLOCK_MAJOR, AEG_ERR_INVALID, "bad slab layout %d", lay);
  AEG_REQUIRE(bytes / sbytes < (1u << 30), AEG_ERR_INVALID, "too many slabs");
  id = pool_id;
  pool_bytes = bytes;
  slab_bytes = sbytes;
  layout = lay;
  n_slabs = uint32_t(bytes / sbytes);
  slabs_.assign(n_slabs, Slab{});
  shapes_.clear();
  qlist_.clear();
  used_ = assigned_ = peak_used_ = peak_assigned_ = 0;
}

int32_t SlabPool::shape_id(const Shape& sh) {
  for (size_t i = 0; i < shapes_.size(); ++i)
    if (shapes_[i] == sh) return int32_t(i);
  shapes_.push_back(sh);
  return int32_t(shapes_.size() - 1);
}

// Reading 6: blocks of already-assigned same-shape slabs first (lowest slab, lowest index), then
// new slabs (lowest index first).  Reading 7: all-or-nothing.
void SlabPool::alloc(const Shape& sh, int32_t n, aeg_block* out) {
  AEG_REQUIRE(n >= 0, AEG_ERR_INVALID, "negative block count");
  const uint32_t kk = k(sh);
  AEG_REQUIRE(kk > 0, AEG_ERR_INVALID, "block of %llu bytes does not fit a %llu-byte slab",
              (unsigned long long)sh.block(), (unsigned long long)slab_bytes);
  if (n == 0) return;
  AEG_REQUIRE(out, AEG_ERR_INVALID, "out is NULL");
  const int32_t sid = shape_id(sh);
  std::vector<aeg_block> got;
  got.reserve(n);
  for (uint32_t s = 0; s < n_slabs && int32_t(got.size()) < n; ++s) {
    Slab& sl = slabs_[s];
    if (sl.shape != sid || sl.n_owned + sl.n_quar >= sl.k) continue;
    for (uint32_t j = 0; j < sl.k && int32_t(got.size()) < n; ++j)
      if (sl.st[j] == 0) got.push_back(make_block(id, s, j));
  }
  std::vector<uint32_t> claimed;
  for (uint32_t s = 0; s < n_slabs && int32_t(got.size()) < n; ++s) {
    if (slabs_[s].shape != -1) continue;
    claimed.push_back(s);
    for (uint32_t j = 0; j < kk && int32_t(got.size()) < n; ++j) got.push_back(make_block(id, s, j));
  }
  if (int32_t(got.size()) < n)
    fail(AEG_ERR_OOM, "pool %d: %d blocks of %llu bytes requested, only %zu available", id, n,
         (unsigned long long)sh.block(), got.size());
  for (uint32_t s : claimed) {
    Slab& sl = slabs_[s];
    sl.shape = sid;
    sl.k = kk;
    sl.st.assign(kk, 0);
    sl.acc.clear();
    sl.acc.resize(kk);
    sl.n_owned = sl.n_quar = 0;
    assigned_ += slab_bytes;
  }
  for (aeg_block b : got) {
    Slab& sl = slabs_[block_slab(b)];
    sl.st[block_idx(b)] = 1;
    sl.n_owned++;
  }
  used_ += uint64_t(n) * sh.block();
  peak_used_ = std::max(peak_used_, used_);
  peak_assigned_ = std::max(peak_assigned_, assigned_);
  std::copy(got.begin(), got.end(), out);
}

void SlabPool::check_owned(const aeg_block* b, int32_t n, const Shape* sh, bool distinct) const {
  AEG_REQUIRE(n >= 0, AEG_ERR_INVALID, "negative block count");
  AEG_REQUIRE(n == 0 || b, AEG_ERR_INVALID, "block array is NULL");
  std::vector<aeg_block> seen;
  if (distinct) seen.assign(b, b + n);
  for (int32_t i = 0; i < n; ++i) {
    const aeg_block h = b[i];
    AEG_REQUIRE(block_pool(h) == id, AEG_ERR_INVALID, "block 0x%llx belongs to pool %d, not %d",
                (unsigned long long)h, block_pool(h), id);
    const uint32_t s = block_slab(h), j = block_idx(h);
    AEG_REQUIRE(s < n_slabs && slabs_[s].shape >= 0 && j < slabs_[s].k, AEG_ERR_INVALID,
                "block 0x%llx outside any assigned slab", (unsigned long long)h);
    if (sh) AEG_REQUIRE(shapes_[slabs_[s].shape] == *sh, AEG_ERR_INVALID, "block 0x%llx has another shape",
                        (unsigned long long)h);
    AEG_REQUIRE(slabs_[s].st[j] == 1, AEG_ERR_STATE, "block 0x%llx is not owned", (unsigned long long)h);
  }
  if (distinct && n > 1) {
    std::sort(seen.begin(), seen.end());
    AEG_REQUIRE(std::adjacent_find(seen.begin(), seen.end()) == seen.end(), AEG_ERR_STATE,
                "repeated block handle");
  }
}

void SlabPool::check_geometry(const aeg_block* b, int32_t n, const Shape& sh) const {
  AEG_REQUIRE(n == 0 || b, AEG_ERR_INVALID, "block array is NULL");
  const uint32_t kk = k(sh);
  AEG_REQUIRE(kk > 0, AEG_ERR_INVALID, "block does not fit the peer's slab");
  for (int32_t i = 0; i < n; ++i)
    AEG_REQUIRE(block_slab(b[i]) < n_slabs && block_idx(b[i]) < kk, AEG_ERR_INVALID,
                "peer block 0x%llx outside the peer pool", (unsigned long long)b[i]);
}

bool SlabPool::busy(aeg_block b, XSet* xs) {
  const Access& a = acc(b);
  bool any = false;
  auto add = [&](uint64_t x) {
    if (x && !done(x)) {
      any = true;
      if (xs) xs->push(x);
    }
  };
  add(a.writer);
  a.readers.each(add);
  return any;
}

void SlabPool::maybe_unassign(uint32_t s) {
  Slab& sl = slabs_[s];
  if (sl.shape >= 0 && sl.n_owned == 0 && sl.n_quar == 0) {  // reading 10
    sl.shape = -1;
    sl.k = 0;
    sl.st.clear();
    sl.acc.clear();
    assigned_ -= slab_bytes;
  }
}

void SlabPool::free(const aeg_block* b, int32_t n) {
  check_owned(b, n, nullptr);
  uint32_t last = UINT32_MAX;
  std::vector<uint32_t> touched;
  for (int32_t i = 0; i < n; ++i) {
    const uint32_t s = block_slab(b[i]), j = block_idx(b[i]);
    Slab& sl = slabs_[s];
    used_ -= shapes_[sl.shape].block();
    sl.n_owned--;
    Access& a = sl.acc[j];
    XSet xs;
    if (busy(b[i], &xs)) {
      sl.st[j] = 2;
      sl.n_quar++;
      a.quar = std::move(xs);
      qlist_.push_back(b[i]);
    } else {
      sl.st[j] = 0;
      a = Access{};
    }
    if (s != last) touched.push_back(last = s);
  }
  for (uint32_t s : touched) maybe_unassign(s);
}

void SlabPool::free_after(const aeg_block* b, int32_t n, uint64_t x) {
  check_owned(b, n, nullptr);
  if (!x || is_done(x)) {
    free(b, n);
    return;
  }
  for (int32_t i = 0; i < n; ++i) {
    const uint32_t s = block_slab(b[i]), j = block_idx(b[i]);
    Slab& sl = slabs_[s];
    used_ -= shapes_[sl.shape].block();
    sl.n_owned--;
    XSet xs;
    busy(b[i], &xs);
    xs.push(x);
    sl.st[j] = 2;
    sl.n_quar++;
    sl.acc[j].quar = std::move(xs);
    qlist_.push_back(b[i]);
  }
}

uint64_t SlabPool::reclaim() {
  uint64_t released = 0;
  std::vector<uint32_t> touched;
  for (size_t q = 0; q < qlist_.size();) {
    const aeg_block blk = qlist_[q];
    Access& a = acc(blk);
    bool all = true;
    a.quar.each([&](uint64_t x) { all = all && done(x); });
    if (!all) {
      ++q;
      continue;
    }
    const uint32_t s = block_slab(blk), j = block_idx(blk);
    slabs_[s].st[j] = 0;
    slabs_[s].n_quar--;
    a = Access{};
    touched.push_back(s);
    qlist_[q] = qlist_.back();  // unordered: swap-pop
    qlist_.pop_back();
    ++released;
  }
  std::sort(touched.begin(), touched.end());
  touched.erase(std::unique(touched.begin(), touched.end()), touched.end());
  for (uint32_t s : touched) maybe_unassign(s);
  return released;
}

// (consecutive blocks usually share their last transfer: skip immediate repeats; callers dedupe)
void SlabPool::deps_for_read(aeg_block b, std::vector<uint64_t>& deps) {
  const Access& a = acc(b);
  if (a.writer && (deps.empty() || deps.back() != a.writer) && !done(a.writer)) deps.push_back(a.writer);
}

void SlabPool::deps_for_write(aeg_block b, std::vector<uint64_t>& deps) {
  const Access& a = acc(b);
  if (a.writer && (deps.empty() || deps.back() != a.writer) && !done(a.writer)) deps.push_back(a.writer);
  a.readers.each([&](uint64_t r) {
    if ((deps.empty() || deps.back() != r) && !done(r)) deps.push_back(r);
  });
}

void SlabPool::note_read(aeg_block b, uint64_t x) {
  Access& a = acc(b);
  a.readers.erase_if([&](uint64_t y) { return done(y); });
  a.readers.push(x);
}

void SlabPool::note_write(aeg_block b, uint64_t x) {
  Access& a = acc(b);
  a.writer = x;
  a.readers.clear();
}

void SlabPool::stats(aeg_pool_stats* o) const {
  *o = aeg_pool_stats{};
  o->pool_bytes = pool_bytes;
  o->slab_bytes = slab_bytes;
  o->n_slabs = n_slabs;
  o->used_bytes = used_;
  o->assigned_bytes = assigned_;
  o->peak_used_bytes = peak_used_;
  o->peak_assigned_bytes = peak_assigned_;
  std::vector<aeg_shape_stats> per(shapes_.size());
  for (size_t i = 0; i < shapes_.size(); ++i) per[i].shape = shapes_[i].to_c();
  for (const Slab& sl : slabs_) {
    if (sl.shape < 0) {
      o->free_slabs++;
      continue;
    }
    per[sl.shape].slabs++;
    per[sl.shape].owned_blocks += sl.n_owned;
    per[sl.shape].quarantined_blocks += sl.n_quar;
    o->owned_blocks += sl.n_owned;
    o->quarantined_blocks += sl.n_quar;
  }
  for (const auto& p : per) {
    if (!p.slabs || o->n_shapes >= 16) continue;
    o->per_shape[o->n_shapes++] = p;
  }
}

}  // namespace aeg
