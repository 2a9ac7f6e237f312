"""Dev: time vpic_load_interpolator (warm, CUDA events) on a configs[] grid."""
import sys
sys.path.insert(0, ".")
import torch
from paper_conf_sc_tanlta25_b200 import inputs, vpic
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 1
wl = inputs.config(cfg)
g = wl.grid
ctx = vpic.Context(g)
fd = torch.from_numpy(inputs.make_fields(g, 0.01)).cuda()
interp = torch.zeros((g.nv, 24), device="cuda")
for _ in range(5):
    vpic.vpic_load_interpolator(ctx, fd, interp)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(50):
    vpic.vpic_load_interpolator(ctx, fd, interp)
e1.record()
torch.cuda.synchronize()
print("load_interpolator (+ghost fill) %.1f us" % (e0.elapsed_time(e1) / 50 * 1e3))
