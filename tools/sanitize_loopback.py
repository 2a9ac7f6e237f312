"""One loopback PIC step through the single-round, device-initiated exchange
(every periodic face routed through the self peer) plus one through the NCCL
face rounds, small enough for compute-sanitizer (tools/sanitize.sh)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_sc_tanlta25_b200 import inputs  # noqa: E402
from paper_conf_sc_tanlta25_b200.pic import HotPath  # noqa: E402

g = inputs.GridSpec(8, 6, 5, dt=0.5, pbc=(0, 0, 1, 0, 0, 1))
wl = inputs.Workload("san", g, [inputs.Species("electron", -1.0, 1.0, 0.6),
                                inputs.Species("ion", 1.0, 4.0, 0.3)], 16, 2, 2)
parts = inputs.make_species_particles(wl)
fields = inputs.make_fields(g, 0.05)
for dev, single in ((True, True), (False, False), (True, False)):
    hp = HotPath(wl, parts, fields, loopback_exchange=True, device_exchange=dev, single_round=single,
                 inbox_cap=4096, capacity_factor=1.0, field_solve=True)
    hp.cycle(2)
    torch.cuda.synchronize()
    print("ok", dev, single, [s.np for s in hp.species])
    hp.close()
