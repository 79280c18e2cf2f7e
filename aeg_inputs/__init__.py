"""Seeded synthetic input generators shared by the oracle-side tests and the CUDA-side tests/bench.

This module holds NONE of the method's arithmetic (no addressing, no allocation, no
sharding, no copy semantics).  It only produces inputs:

* request lengths, churn sequences and placement decisions (PCG64, seed = 1000 + config id),
* KV / weight *content* via a counter-based generator (splitmix64 of a 64-bit key), so that
  any byte of any synthetic pool can be regenerated from its key without materialising pools,
* model tensor lists (public HF config shapes; sizes only, content is synthetic).

The counter-based generator exists twice, as the task rules allow: in NumPy (`gen.py`) and in
CUDA/C (`csrc/inputs.cu`, built into `libaeginputs.so`).  Their agreement is tested
(`tests/test_inputs.py`, `tests/test_gpu_inputs.py`).
"""
from .gen import *  # noqa: F401,F403
