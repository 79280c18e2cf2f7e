// Unified KV cache: slab allocator with move-list quarantine (H1).
//
// PAPER.md:1369-1381 (§5.2): every KV region (VRAM or DRAM) is cut into fixed-size slabs; each
// slab is assigned one shape and serves as a pool of blocks of that shape; allocation first uses
// free blocks of same-shape slabs, then acquires new slabs; freeing returns blocks to their slab
// and reclaims slabs with no occupied blocks.  PAPER.md:1553-1562 (§5.3): blocks touched by
// in-flight copies sit in move lists that allocation neglects (rule ❸) until a daemon observes
// their events complete (step ⑧).  Readings 6-10 in DESIGN.md fix the unspecified choices.
//
// Pure host logic (no CUDA); the owning context supplies transfer completion (is_done).
#pragma once

#include <algorithm>
#include <functional>
#include <memory>
#include <vector>

#include "common.h"

namespace aeg {

class SlabPool {
 public:
  // A small set of transfer ids: two inline, the rest on the heap (a block rarely has more than
  // one or two in-flight readers or move-list transfers).
  struct XSet {
    uint64_t a = 0, b = 0;
    std::unique_ptr<std::vector<uint64_t>> rest;
    XSet() = default;
    XSet(XSet&&) = default;
    XSet& operator=(XSet&&) = default;
    XSet(const XSet& o) : a(o.a), b(o.b), rest(o.rest ? new std::vector<uint64_t>(*o.rest) : nullptr) {}
    XSet& operator=(const XSet& o) {
      if (this != &o) {
        a = o.a;
        b = o.b;
        rest.reset(o.rest ? new std::vector<uint64_t>(*o.rest) : nullptr);
      }
      return *this;
    }
    void push(uint64_t x) {
      if (!a) a = x;
      else if (!b) b = x;
      else {
        if (!rest) rest.reset(new std::vector<uint64_t>());
        rest->push_back(x);
      }
    }
    template <class F> void each(F f) const {
      if (a) f(a);
      if (b) f(b);
      if (rest)
        for (uint64_t x : *rest) f(x);
    }
    template <class P> void erase_if(P pred) {
      if (a && pred(a)) a = 0;
      if (b && pred(b)) b = 0;
      if (!a && b) std::swap(a, b);
      if (rest) {
        rest->erase(std::remove_if(rest->begin(), rest->end(), pred), rest->end());
        while (!rest->empty() && (!a || !b)) {
          (!a ? a : b) = rest->back();
          rest->pop_back();
        }
        if (rest->empty()) rest.reset();
      }
    }
    bool empty() const { return !a && !b && !rest; }
    void clear() {
      a = b = 0;
      rest.reset();
    }
  };
  struct Access {     // per-block last access, for rules ❷❸, and its move-list transfers
    uint64_t writer = 0;  // last transfer that wrote the block (0 = none)
    XSet readers;         // transfers that read it since that write
    XSet quar;            // move list (st == 2): transfers that must complete before reuse
  };

  void init(int pool_id, uint64_t pool_bytes, uint64_t slab_bytes, int layout);

  int id = 0;
  uint64_t pool_bytes = 0, slab_bytes = 0;
  int layout = AEG_LAYER_MAJOR;
  uint32_t n_slabs = 0;
  std::function<bool(uint64_t)> is_done;  // transfer id -> completion observed
  // Owner-maintained watermark: every transfer id below it has completed (fast path of done()).
  const uint64_t* done_below = nullptr;
  bool done(uint64_t x) const { return (done_below && x < *done_below) || is_done(x); }

  uint32_t k(const Shape& sh) const { return uint32_t(slab_bytes / sh.block()); }
  // Byte offset (from the pool base) of layer 0 of block b, and the per-layer stride:
  //   layer-major  addr = s*S + l*k*Cl + j*Cl      block-major  addr = s*S + j*L*Cl + l*Cl
  uint64_t off0(aeg_block b, const Shape& sh) const {
    uint64_t base = uint64_t(block_slab(b)) * slab_bytes;
    return layout == AEG_LAYER_MAJOR ? base + uint64_t(block_idx(b)) * sh.chunk()
                                     : base + uint64_t(block_idx(b)) * sh.block();
  }
  uint64_t lstride(const Shape& sh) const {
    return layout == AEG_LAYER_MAJOR ? uint64_t(k(sh)) * sh.chunk() : sh.chunk();
  }

  // H1 API.  alloc/free validate everything before changing state (all-or-nothing).
  void alloc(const Shape& sh, int32_t n, aeg_block* out);
  void free(const aeg_block* b, int32_t n);
  // free, keeping the blocks in the move list until transfer `x` (too) has completed
  void free_after(const aeg_block* b, int32_t n, uint64_t x);
  uint64_t reclaim();  // release move-list blocks whose transfers all completed
  // Validate that b[0..n) are distinct owned blocks of this pool (and of shape sh if given).
  void check_owned(const aeg_block* b, int32_t n, const Shape* sh, bool distinct = true) const;
  // Validate handles against the geometry only (peer pools): slab in range, index < k(sh).
  void check_geometry(const aeg_block* b, int32_t n, const Shape& sh) const;
  void stats(aeg_pool_stats* out) const;
  uint64_t quarantined() const { return qlist_.size(); }

  // Rule ❷❸ bookkeeping: incomplete transfers a new access must wait for.  The blocks must be
  // owned blocks of this pool (callers validate with check_owned first).
  void deps_for_read(aeg_block b, std::vector<uint64_t>& deps);
  void deps_for_write(aeg_block b, std::vector<uint64_t>& deps);
  void note_read(aeg_block b, uint64_t x);
  void note_write(aeg_block b, uint64_t x);
  void forget_completed() {}  // completed ids are dropped lazily (note_read) or on free / reclaim

 private:
  // Per slab, flat per-block arrays sized k when the slab is assigned to a shape: O(1) state and
  // last-access lookups by (slab, index), no hashing and no per-block heap nodes on the data path.
  struct Slab {
    int32_t shape = -1;          // index into shapes_, -1 = unassigned
    uint32_t k = 0, n_owned = 0, n_quar = 0;
    std::vector<uint8_t> st;     // 0 free, 1 owned, 2 quarantined (move list)
    std::vector<Access> acc;     // per block
  };
  Access& acc(aeg_block b) { return slabs_[block_slab(b)].acc[block_idx(b)]; }
  int32_t shape_id(const Shape& sh);
  bool busy(aeg_block b, XSet* xs);
  void maybe_unassign(uint32_t s);

  std::vector<Slab> slabs_;
  std::vector<Shape> shapes_;
  std::vector<aeg_block> qlist_;  // blocks in the move list (st == 2), unordered
  uint64_t used_ = 0, assigned_ = 0, peak_used_ = 0, peak_assigned_ = 0;
};

}  // namespace aeg
