"""Model of the current scatter's L2 reductions per particle vs steps since
the sort (C2 electrons: u_th = 0.1, c dt = 0.548, 128 ppc, chunks of 64 taken
from one voxel): the current warp deposit (segments >= MIN_SEG summed, 12
red.f32 ~ 4 red.v4; other items 3 red.v4 each) against an idealised one that
sorts G consecutive particles by current voxel and pays 3 red.v4 per distinct
voxel of every 32-lane set.  Dev tool.

    python tools/sim_reductions.py
"""
import numpy as np

rng = np.random.default_rng(1)
SIGMA_PER_STEP = 0.1 * 0.548 / np.sqrt(1.0 + 3 * 0.01)   # thermal displacement per axis per step


def sim(t, group, trials=300, min_seg=7):
    s = SIGMA_PER_STEP * t
    cur = srt = n = 0
    for _ in range(trials):
        off = rng.uniform(-0.5, 0.5, (group, 3)) + rng.normal(0, s, (group, 3))
        v = np.floor(off + 0.5).astype(int)
        key = v[:, 0] + 100 * v[:, 1] + 10000 * v[:, 2]
        for c in range(0, group, 64):
            a, b = key[c:c + 32], key[c + 32:c + 64]
            u, cnt = np.unique(np.concatenate([a, b]), return_counts=True)
            for kk, cc in zip(u, cnt):
                big = (a == kk).sum() >= min_seg or (b == kk).sum() >= min_seg
                cur += 4 if big else 3 * cc
        ks = np.sort(key)
        for c in range(0, group, 32):
            srt += 3 * len(np.unique(ks[c:c + 32]))
        n += group
    return cur / n, srt / n


if __name__ == "__main__":
    print("steps_since_sort  current  sorted64  sorted128  sorted256   (red.v4 per particle)")
    for t in (0, 2, 5, 10, 15, 19):
        c, s64 = sim(t, 64)
        _, s128 = sim(t, 128)
        _, s256 = sim(t, 256)
        print(f"{t:16d}  {c:7.2f}  {s64:8.2f}  {s128:9.2f}  {s256:9.2f}")
