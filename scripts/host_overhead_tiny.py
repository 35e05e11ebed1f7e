"""Fixed per-call host overhead of load() / enumerate() / free() (wall, medians over 50 calls) on a
tiny graph and on gh_work, next to the enumeration kernel's device time."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config, g0_edges  # noqa: E402

for name in ["g0", "gh_work"]:
    nu, nv, e = g0_edges() if name == "g0" else make_config(name)
    ed = torch.from_numpy(np.asarray(e).astype("int32")).cuda()
    s = torch.cuda.current_stream()
    tl, te, tf, tk, tev = [], [], [], [], []
    for it in range(50 if name == "g0" else 10):
        torch.cuda.synchronize()
        a0 = torch.cuda.Event(enable_timing=True)
        a1 = torch.cuda.Event(enable_timing=True)
        a0.record(s)
        t0 = time.perf_counter()
        g = gmbe.load(nu, nv, ed, stream=s)
        t1 = time.perf_counter()
        r = g.enumerate(stream=s)
        t2 = time.perf_counter()
        g.free()
        t3 = time.perf_counter()
        a1.record(s)
        a1.synchronize()
        if it >= 2:
            tl.append(1e3 * (t1 - t0)); te.append(1e3 * (t2 - t1)); tf.append(1e3 * (t3 - t2)); tk.append(r.kernel_ms)
            tev.append(a0.elapsed_time(a1))
    med = statistics.median
    print("%-8s load %.3f  enumerate %.3f  free %.3f  (kernel %.3f)  device-timed step %.3f ms" % (
        name, med(tl), med(te), med(tf), med(tk), med(tev)), flush=True)
