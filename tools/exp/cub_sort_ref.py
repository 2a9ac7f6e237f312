import torch, time
n = 1 << 28
k = torch.randint(0, 2197000, (n,), dtype=torch.int32, device="cuda")
k, _ = torch.sort(k)           # nearly sorted like ours? make it sorted then perturb
k = (k + torch.randint(-16900, 16901, (n,), dtype=torch.int32, device="cuda").clamp(-1, 1) * torch.randint(0, 2, (n,), dtype=torch.int32, device="cuda")).clamp(0, 2196999)
for stable in (True,):
    for rep in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); v, i = torch.sort(k, stable=stable); e1.record(); torch.cuda.synchronize()
        print("torch.sort int32 keys + int64 idx, n=2^28:", round(e0.elapsed_time(e1), 3), "ms")
