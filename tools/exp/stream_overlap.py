"""Dev: the two species' advance_p on two streams with the full 2 CTAs/SM
each (the second kernel's CTAs fill the first's tail) vs one stream; and the
CUDA-graph period.  Default C2 bench otherwise."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
mode = sys.argv[1]
sys.argv = ["bench.py", "--steps", "3", "--warmup", "2", "--no-e2e", "--no-cpu-baseline"] + \
    (["--concurrent-species"] if mode in ("conc1", "conc2") else [])
import paper_conf_sc_tanlta25_b200.pic as P  # noqa: E402
from paper_conf_sc_tanlta25_b200 import vpic  # noqa: E402

orig = P.HotPath.__init__


def init(self, *a, **kw):
    if mode == "graphs":
        kw["graphs"] = True
    orig(self, *a, **kw)
    if mode == "conc2":
        self.ctx.set_option(vpic.VPIC_OPT_ADVANCE_CTAS_PER_SM, 0)


P.HotPath.__init__ = init
import bench  # noqa: E402
bench.main()
