"""Fig. 6 analogue: gather-scatter
bandwidth on B200 for the paper's three key patterns and three sort orders.

* n = 1e9 doubles; keys: contiguous unique (nkeys = n), repeated (1e7 keys x
  100), 5-point stencil on a 3163-wide 2-D index (1e7 keys x 100);
* orders of the repeated / stencil keys: standard (sorted), strided (Alg. 1:
  lexicographic (r, k)), tiled strided (Alg. 2: (floor(k/T), r, k),
  T = 3 x SMs x 128), random (seeded shuffle) -- generated directly in those
  orders (they are permutations of "every key 100 times");
* bandwidth = algorithmic bytes / median kernel time, bytes = n (4 key + 8 x +
  8 out) + n P (8 gather + 8 scatter), P = 1 or 5 access points (reading F2);
* scatter: per-lane FP64 atomics (the paper's kernel) and warp-aggregated.

    python tools/gather_scatter_bench.py [--n 1000000000] > profiles/..jsonl
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs, vpic  # noqa: E402


def make_keys(n, K, m, order, T, dev):
    i = torch.arange(n, device=dev, dtype=torch.int64)
    if order == "standard":
        k = i // m
    elif order == "strided":
        k = i % K
    elif order == "tiled_strided":
        c = i // (T * m)
        w = torch.clamp(K - c * T, max=T)              # width of the chunk (last one partial)
        j = i - c * T * m
        k = c * T + j % w
    else:  # random
        g = torch.Generator(device=dev)
        g.manual_seed(11)
        k = (i // m)[torch.randperm(n, device=dev, generator=g)]
    return k.to(torch.int32)


def timed(fn, reps=5):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    fn()
    fn()
    torch.cuda.synchronize()
    for a, b in ev:
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    t = sorted(a.elapsed_time(b) for a, b in ev)
    return t[len(t) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1_000_000_000)
    args = ap.parse_args()
    dev = torch.device("cuda")
    vpic.load()
    ctx = vpic.Context(inputs.GridSpec(4, 4, 4))
    sms = ctx.info()["num_sms"]
    T = 3 * sms * 128
    n = args.n
    x = torch.rand(n, device=dev, dtype=torch.float64)
    out = torch.empty_like(x)
    cases = [("contiguous", n, 1, 0, ["standard"])]
    K, m = n // 100, 100
    nx = 3163
    cases += [("repeated", K, m, 0, ["standard", "strided", "tiled_strided", "random"]),
              ("stencil5", K, m, nx, ["standard", "strided", "tiled_strided", "random"])]
    for name, nkeys, mult, snx, orders in cases:
        table = torch.rand(nkeys, device=dev, dtype=torch.float64)
        acc = torch.zeros(nkeys, device=dev, dtype=torch.float64)
        P = 5 if snx else 1
        nbytes = n * (4 + 8 + 8) + n * P * 16
        for order in orders:
            keys = torch.arange(n, device=dev, dtype=torch.int32) if name == "contiguous" else \
                make_keys(n, nkeys, mult, order, T, dev)
            for agg in (0, 1):
                ms = timed(lambda: vpic.vpic_gather_scatter(ctx, keys, x, table, out, acc, snx, agg))
                print(json.dumps({"pattern": name, "order": order, "scatter": "warp" if agg else "lane",
                                  "n": n, "nkeys": nkeys, "access_points": P, "ms": ms,
                                  "GBps": nbytes / ms / 1e6, "tile_sz": T}), flush=True)
            del keys
            torch.cuda.empty_cache()
        del table, acc


if __name__ == "__main__":
    main()
