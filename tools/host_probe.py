"""Tuning aid: wall time of dt_pack_host / dt_unpack_host on C2 with pinned buffers,
under the current DT_HOST_PIPE / DT_HOST_CHUNK settings."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from workloads import c2_lower_triangle, fill_bytes  # noqa: E402

rec, org, parent = c2_lower_triangle()
t = dt.from_recipe(rec).commit()
src = torch.from_numpy(fill_bytes(parent, 3)).pin_memory()
dst = torch.full((parent,), 0xA5, dtype=torch.uint8).pin_memory()
pk = torch.empty(t.size, dtype=torch.uint8).pin_memory()
for name, fn in (("pack_host", lambda: dt.pack_host(t, 1, src.data_ptr() + org, pk.data_ptr(), stream=0)),
                 ("unpack_host", lambda: dt.unpack_host(t, 1, pk.data_ptr(), dst.data_ptr() + org, stream=0))):
    for _ in range(2):
        fn()
    ts = []
    for _ in range(8):
        t0 = time.perf_counter()
        fn()
        ts.append(time.perf_counter() - t0)
    print(f"{os.environ.get('DT_HOST_PIPE', '1')} chunk={os.environ.get('DT_HOST_CHUNK', 'def')} {name}: "
          f"{min(ts) * 1e3:.3f} ms  {2 * t.size / min(ts) / 1e9:.1f} GB/s (H2D+D2H)")
