"""Host wall time of load() and enumerate() vs the enumeration kernel's device time, per call."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    ed = torch.from_numpy(e.astype("int32")).cuda()
    for it in range(5):
        t0 = time.perf_counter()
        g = gmbe.load(nu, nv, ed)
        t1 = time.perf_counter()
        r = g.enumerate()
        t2 = time.perf_counter()
        g.free()
        print(name, it, "load %.2f ms  enumerate %.2f ms  kernel %.2f ms" % (1e3 * (t1 - t0), 1e3 * (t2 - t1), r.kernel_ms), flush=True)
