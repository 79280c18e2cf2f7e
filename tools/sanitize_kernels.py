"""Drive the round-2 kernel paths outside pytest (compute-sanitizer racecheck / synccheck cannot run
under the pytest process): C1 round trips with every kernel and layout pair, small shapes, local
migrates (AUTO = BULKW) — each checked against the oracle by the test bodies themselves."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402
from tests import test_gpu_edges as E  # noqa: E402
from tests import test_gpu_migrate as M  # noqa: E402
from tests import test_gpu_swap as S  # noqa: E402

n = 0
for k in (aeg.KERNEL_BULKW, aeg.KERNEL_BULK, aeg.KERNEL_LSU, aeg.KERNEL_WARP):
    for lay in S.LAYOUTS:
        S.test_c1_round_trip_full_images(lay, k, 1 << 20)
        n += 1
for shape in [(1, 1, 8, 2, 1), (3, 1, 8, 2, 1), (1, 2, 64, 2, 16)]:
    for k in (aeg.KERNEL_AUTO, aeg.KERNEL_BULKW):
        E.test_small_shapes_round_trip(shape, k)
        n += 1
for k in (aeg.KERNEL_AUTO, aeg.KERNEL_BULKW):
    for ce in (False, True):          # fused kernel / copy-engine route
        M.test_local_migrate(k, ce)
        n += 1
print(f"{n} oracle-checked cases passed")
