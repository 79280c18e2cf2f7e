import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

# GPU files run cheapest-parity-first, so that under -x a failure in a heavy test (full-size pools,
# multi-process IPC, race stress) cannot hide the C1 parity results; everything else keeps its order.
_GPU_ORDER = ["test_gpu_swap.py", "test_gpu_dma_edges.py", "test_c_client.py", "test_gpu_edges.py", "test_gpu_fuzz.py", "test_gpu_shapes.py", "test_gpu_weights.py",
              "test_gpu_switch.py", "test_gpu_migrate.py", "test_gpu_dist.py", "test_gpu_stress.py", "test_gpu_c5.py",
              "test_gpu_fullsize.py"]


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a); run with -m gpu")
    config.addinivalue_line("markers", "slow: long CPU test")


def pytest_collection_modifyitems(config, items):
    # GPU tests must not silently pass without a GPU: they fail loudly when selected and no GPU
    # is present (the product path has no CPU fallback).
    def key(it):
        name = os.path.basename(str(it.fspath))
        return _GPU_ORDER.index(name) if name in _GPU_ORDER else -1
    items.sort(key=key)     # stable: non-GPU files (-1) first, in collection order


@pytest.fixture(scope="session")
def _built_from_source():
    """Compile libaegkv.so and libaeginputs.so from the checked-out sources once per session
    (forced: a box must never run binaries built elsewhere)."""
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    # AEG_TESTS_NO_REBUILD=1: keep the in-tree build (compute-sanitizer runs, which would otherwise
    # follow nvcc's child processes)
    return build.build(force=os.environ.get("AEG_TESTS_NO_REBUILD") != "1")


@pytest.fixture(autouse=True)
def _gpu_tests_use_fresh_build(request):
    if request.node.get_closest_marker("gpu") is not None:
        request.getfixturevalue("_built_from_source")
