"""O1 — KV shape arithmetic.  TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md:1120-1128 (Table 1): "The shape and size of KV cache for different models in vLLM.
Listed values pertain to a single token in 16-bit precision", shape (L, 2, H, D).
Readings: B = 16 tokens per block (reading 1); a block spans B tokens x all L layers
(reading 2); the per-layer chunk of a block is laid out [2][B][H][D] (reading 3).
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class KVShape:
    L: int          # layers
    H: int          # KV heads (per TP rank)
    D: int          # head dim
    s: int = 2      # bytes per element (16-bit)
    B: int = 16     # tokens per block (reading 1)

    def token_bytes(self) -> int:
        """Table 1 per-token size: product of shape (L, 2, H, D) times s bytes."""
        return self.L * 2 * self.H * self.D * self.s

    def chunk_bytes(self) -> int:
        """Cl: one block's slice of one layer = B tokens x (2, H, D) x s."""
        return self.B * 2 * self.H * self.D * self.s

    def block_bytes(self) -> int:
        """One block across all L layers."""
        return self.L * self.chunk_bytes()

    def blocks_for(self, tokens: int) -> int:
        """Number of blocks holding ``tokens`` tokens: ceil(T / B)."""
        return -(-tokens // self.B)

    def live_tokens(self, tokens: int, j: int) -> int:
        """Live tokens of logical block j of a T-token request: min(B, T - jB) (0 if past end)."""
        return max(0, min(self.B, tokens - j * self.B))

    def elem_offset(self, c: int, slot: int, h: int, d: int) -> int:
        """Byte offset inside a chunk of element (c in {K,V}, token slot, head, dim) — reading 3."""
        return (((c * self.B + slot) * self.H + h) * self.D + d) * self.s

    def as_tuple(self):
        return (self.L, self.H, self.D, self.s, self.B)


def shape_of(t) -> KVShape:
    L, H, D, s, B = t
    return KVShape(L, H, D, s, B)
