"""Tuning aid: event-timed pack/unpack of a few irregular lists under forced kernel
families (DT_FORCE_KERNEL), L2 flushed between reps."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from workloads import c5b_irregular  # noqa: E402


def unsorted_structs(n=1 << 20, seed=5):
    rng = np.random.default_rng(seed)
    rec = ("resized", ("struct", [1, 1], [0, 8], [("basic", "INT32"), ("basic", "DOUBLE")]), 0, 16)
    slots = rng.permutation(2 * n)[:n]
    return ("hindexed", np.ones(n, dtype=np.int64), slots.astype(np.int64) * 16, rec), 0, 2 * n * 16 + 64


def shuffled_c5b(m=64 << 20):
    rec, org, parent = c5b_irregular(m)
    _, lens, disp, base = rec
    rng = np.random.default_rng(9)
    perm = rng.permutation(len(lens))
    return ("hindexed", lens[perm], disp[perm], base), org, parent


def local_shuffle(m=64 << 20, group=48):
    rec, org, parent = c5b_irregular(m)
    _, lens, disp, base = rec
    rng = np.random.default_rng(3)
    n = len(lens) - len(lens) % group
    perm = np.concatenate([rng.permutation(group) + i for i in range(0, n, group)] + [np.arange(n, len(lens))])
    return ("hindexed", lens[perm], disp[perm], base), org, parent


def gran16(m=64 << 20):
    rng = np.random.default_rng(4)
    n = m // 72
    lens = rng.integers(1, 9, n) * 16
    gaps = rng.integers(0, 5, n) * 16
    disp = np.concatenate([[0], np.cumsum(lens[:-1] + gaps[:-1])])
    return ("hindexed", lens, disp, ("basic", "BYTE")), 0, int(disp[-1] + lens[-1])


def main():
    dev = torch.device("cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for name, mk in (("C5b", lambda: c5b_irregular(64 << 20)), ("C5b shuffled", shuffled_c5b),
                     ("C5b shuffled/48", local_shuffle), ("gran16", gran16),
                     ("unsorted structs", unsorted_structs)):
        rec, org, parent = mk()
        t = dt.from_recipe(rec).commit()
        src = torch.randint(0, 255, (parent,), dtype=torch.uint8, device=dev)
        pk = torch.empty(t.size, dtype=torch.uint8, device=dev)
        for kind in ("3", "7"):
            os.environ["DT_FORCE_KERNEL"] = kind
            ts = []
            for r in range(8):
                flush.fill_(r)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                dt.pack(t, 1, src, pk, origin_offset=org)
                e1.record()
                torch.cuda.synchronize()
                if r >= 2:
                    ts.append(e0.elapsed_time(e1) * 1e3)
            print(f"{name:18s} kind {kind}: pack {np.median(ts):8.1f} us  payload {t.size}  "
                  f"(planner: {t.plan(1, src.data_ptr() + org, pk.data_ptr(), 0, t.size)})")
        os.environ.pop("DT_FORCE_KERNEL")


if __name__ == "__main__":
    main()
