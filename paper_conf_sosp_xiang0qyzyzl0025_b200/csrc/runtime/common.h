// Internal helpers shared by the runtime translation units (not part of the ABI).
#pragma once

#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <stdexcept>
#include <string>

#include "aeg.h"

namespace aeg {

// Internal failures are C++ exceptions carrying an AEG_ERR_* code; every extern "C" entry point
// converts them into a return code + thread-local message (capi.cc).  Nothing escapes the ABI.
struct Error : std::runtime_error {
  int code;
  Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

[[noreturn]] inline void fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  throw Error(code, buf);
}

#define AEG_REQUIRE(cond, code, ...) \
  do {                               \
    if (!(cond)) ::aeg::fail(code, __VA_ARGS__); \
  } while (0)

inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// Block handle encoding (aeg.h): [63:62] pool, [61:32] slab, [31:0] index.
inline aeg_block make_block(int pool, uint32_t slab, uint32_t idx) {
  return (uint64_t(pool & 3) << 62) | (uint64_t(slab & 0x3FFFFFFFu) << 32) | idx;
}
inline int block_pool(aeg_block b) { return int(b >> 62); }
inline uint32_t block_slab(aeg_block b) { return uint32_t((b >> 32) & 0x3FFFFFFFu); }
inline uint32_t block_idx(aeg_block b) { return uint32_t(b & 0xFFFFFFFFu); }

// KV shape: (L, 2, H, D) x s bytes per token, B tokens per block (Table 1).
struct Shape {
  int32_t L = 0, H = 0, D = 0, s = 0, B = 0;
  static Shape from(const aeg_kv_shape* p) {
    AEG_REQUIRE(p, AEG_ERR_INVALID, "shape is NULL");
    Shape x{p->num_layers, p->num_kv_heads, p->head_dim, p->elem_bytes, p->block_tokens};
    AEG_REQUIRE(x.L > 0 && x.H > 0 && x.D > 0 && x.s > 0 && x.B > 0 && x.L <= 4096, AEG_ERR_INVALID,
                "shape fields must be positive (L=%d H=%d D=%d s=%d B=%d)", x.L, x.H, x.D, x.s, x.B);
    AEG_REQUIRE(x.chunk() % 16 == 0, AEG_ERR_INVALID, "chunk bytes %llu not a multiple of 16",
                (unsigned long long)x.chunk());
    return x;
  }
  uint64_t chunk() const { return uint64_t(B) * 2 * H * D * s; }  // Cl: one block, one layer
  uint64_t block() const { return chunk() * uint64_t(L); }         // one block, all layers
  bool operator==(const Shape& o) const {
    return L == o.L && H == o.H && D == o.D && s == o.s && B == o.B;
  }
  aeg_kv_shape to_c() const { return aeg_kv_shape{L, H, D, s, B}; }
};

}  // namespace aeg
