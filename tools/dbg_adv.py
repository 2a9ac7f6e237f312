import sys, torch, numpy as np
sys.path.insert(0, '.')
from paper_conf_sc_tanlta25_b200 import inputs, vpic
vpic.load()
n = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
g = inputs.GridSpec(16, 16, 16)
p = inputs.random_particles(g, n, 1, u_scale=0.3)
p = p[np.argsort(p["i"], kind="stable")]
ctx = vpic.Context(g)
ctx.set_option(vpic.VPIC_OPT_ADVANCE_KERNEL, 2)
ctx.set_option(vpic.VPIC_OPT_DEPOSIT, 2)
fd = torch.from_numpy(inputs.make_fields(g, 0.01)).cuda()
interp = torch.zeros((g.nv, 24), device="cuda")
vpic.vpic_load_interpolator(ctx, fd, interp)
acc = torch.zeros((g.nv, 12), device="cuda")
pd = vpic.particles_to_device(p)
nm = torch.zeros(1, dtype=torch.int64, device="cuda")
mv = torch.zeros((1024, 4), device="cuda")
vpic.vpic_advance_p(ctx, -1.0, 1.0, pd, n, interp, acc, mv, 1024, nm, None)
torch.cuda.synchronize()
print("ok", n)
