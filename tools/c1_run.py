"""C1 (BASELINE configs[0]) ops through the API on one arena, for ncu launch lists of the
small-op regime:  ncu --metrics gpu__time_duration.sum -k regex:'^k_' python tools/c1_run.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402,F401

import tracegen as tg  # noqa: E402
from paper_conf_iiswc_zhucvhcr22_b200 import build, harness, um  # noqa: E402

build.build()
t = tg.gen_c1(0)
a = harness.make_arena(t, "eager", flags=um.UM_F_APP_STAMP)
harness.issue(a, t, "eager", 0, int(sys.argv[1]) if len(sys.argv) > 1 else 1000)
print(um.um_get_stats(a.handle))
a.close()
