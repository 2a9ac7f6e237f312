"""Dev: pinned host <-> device copy bandwidth on the GPU box (PCIe), the e2e bound.
    python tools/pcie_bw.py [--bind]   (--bind: pin the process to the GPU's local CPUs first)"""
import os, sys, time
if "--bind" in sys.argv:
    sys.path.insert(0, ".")
    from paper_conf_sc_tanlta25_b200.pic import bind_to_gpu_cpus
    print("bound to", bind_to_gpu_cpus(0))
print("cpus", len(os.sched_getaffinity(0)), sorted(os.sched_getaffinity(0))[:4], "...")
import torch
n = 8 * (1 << 30) // 4  # 8 GiB floats
h = torch.empty(n, dtype=torch.float32).pin_memory()
h2 = torch.empty(n, dtype=torch.float32).pin_memory()
d = torch.empty(n, dtype=torch.float32, device="cuda")
d2 = torch.empty(n, dtype=torch.float32, device="cuda")
def timeit(fn, reps=3):
    fn(); torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) / reps
B = n * 4
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
print("h2d 1 stream GB/s", B / timeit(lambda: d.copy_(h, non_blocking=True)) / 1e9)
print("d2h 1 stream GB/s", B / timeit(lambda: h.copy_(d, non_blocking=True)) / 1e9)
def two():
    with torch.cuda.stream(s1): d[: n // 2].copy_(h[: n // 2], non_blocking=True)
    with torch.cuda.stream(s2): d[n // 2:].copy_(h[n // 2:], non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1); torch.cuda.current_stream().wait_stream(s2)
print("h2d 2 streams GB/s", B / timeit(two) / 1e9)
def chunks():
    c = 1 << 26
    for i in range(0, n, c): d[i:i + c].copy_(h[i:i + c], non_blocking=True)
print("h2d 256MB chunks GB/s", B / timeit(chunks) / 1e9)
def bidir():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1); torch.cuda.current_stream().wait_stream(s2)
t = timeit(bidir)
print("bidir each way GB/s", B / t / 1e9)
