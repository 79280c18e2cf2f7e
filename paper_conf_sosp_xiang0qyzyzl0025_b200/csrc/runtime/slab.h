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

#include <functional>
#include <unordered_map>
#include <vector>

#include "common.h"

namespace aeg {

class SlabPool {
 public:
  struct Access {                 // per-block last access, for rules ❷❸
    uint64_t writer = 0;          // last transfer that wrote the block (0 = none)
    std::vector<uint64_t> readers;  // transfers that read it since that write
  };

  void init(int pool_id, uint64_t pool_bytes, uint64_t slab_bytes, int layout);

  int id = 0;
  uint64_t pool_bytes = 0, slab_bytes = 0;
  int layout = AEG_LAYER_MAJOR;
  uint32_t n_slabs = 0;
  std::function<bool(uint64_t)> is_done;  // transfer id -> completion observed

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
  uint64_t quarantined() const { return quarantine_.size(); }

  // Rule ❷❸ bookkeeping: incomplete transfers a new access must wait for.
  void deps_for_read(aeg_block b, std::vector<uint64_t>& deps);
  void deps_for_write(aeg_block b, std::vector<uint64_t>& deps);
  void note_read(aeg_block b, uint64_t x);
  void note_write(aeg_block b, uint64_t x);
  void forget_completed();  // drop access entries whose transfers completed

 private:
  struct Slab {
    int32_t shape = -1;          // index into shapes_, -1 = unassigned
    uint32_t k = 0, n_owned = 0, n_quar = 0;
    std::vector<uint8_t> st;     // 0 free, 1 owned, 2 quarantined (move list)
  };
  int32_t shape_id(const Shape& sh);
  bool busy(aeg_block b, std::vector<uint64_t>* xs);
  void maybe_unassign(uint32_t s);

  std::vector<Slab> slabs_;
  std::vector<Shape> shapes_;
  std::unordered_map<aeg_block, std::vector<uint64_t>> quarantine_;  // move list: block -> xfers
  std::unordered_map<aeg_block, Access> access_;
  uint64_t used_ = 0, assigned_ = 0, peak_used_ = 0, peak_assigned_ = 0;
};

}  // namespace aeg
