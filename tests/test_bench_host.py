"""Host-side logic of bench.py that needs no GPU: the paper-context block, the argument defaults the
driver relies on, the GPU-local core parser and the Dist helpers at world size 1."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_paper_context_tolerates_missing_legs_and_picks_ours():
    empty = bench.paper_context({})
    assert empty["auto_scaling_latency"]["ours_llama7b_switch_ms_p50"] == {"staged": None, "direct": None,
                                                                           "prefetch": None}
    out = {"switch": {"staged": {"per_model": {"llama-7b": {"last_layer_ms_p50": 277.0, "h2d_GBps": 52.0}}}},
           "per_request_sync": {"overhead_vs_memcpy_ms_p50": 3.0, "overhead_vs_memcpy_ms_max": 5.0}}
    c = bench.paper_context(out)
    assert c["auto_scaling_latency"]["ours_llama7b_switch_ms_p50"]["staged"] == 277.0
    assert c["kv_sync_overhead_per_request"]["ours_overhead_vs_memcpy_ms_p50_max"] == [3.0, 5.0]
    assert c["weight_load_bandwidth"]["ours_staged_llama7b_h2d_GBps"] == 52.0
    assert "PAPER.md:2020-2025" in c["auto_scaling_latency"]["paper"]


def test_defaults_are_the_driver_contract(monkeypatch):
    monkeypatch.setattr(sys, "argv", ["bench.py"])
    a = bench.parse()
    assert a.gpus == 1 and a.impl != "reference" and a.steps >= 1 and a.warmup >= 3
    assert not a.probe_peer_bulk          # the peer bulk-store probe is opt-in
    monkeypatch.setattr(sys, "argv", ["bench.py", "--impl", "reference", "--gpus", "2", "--steps", "3",
                                      "--warmup", "3"])
    a = bench.parse()
    assert a.impl == "reference" and a.gpus == 2 and a.steps == 3


def test_single_rank_dist_helpers_need_no_process_group():
    d = bench.Dist.__new__(bench.Dist)   # the world-size-1 paths never touch torch.distributed
    d.world, d.rank, d.local = 1, 0, 0
    assert d.max(2.5) == 2.5 and d.sum(3.0) == 3.0 and d.gather_obj({"a": 1}) == [{"a": 1}]


def test_gpu_local_cpus_is_none_or_a_cpu_set():
    cpus = bench.gpu_local_cpus()
    assert cpus is None or (isinstance(cpus, set) and all(isinstance(c, int) and c >= 0 for c in cpus))
    with bench.one_core() as pin:
        if hasattr(os, "sched_getaffinity"):
            assert len(os.sched_getaffinity(0)) == 1
    assert set(pin.describe()) == {"core_id", "on_gpu_numa_node"}
