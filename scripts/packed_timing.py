"""Timing of snicit_infer_packed by bits source (device / pinned host / pageable host) on C2."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork, pack_rows  # noqa: E402
from workload import sdgc  # noqa: E402

N, L, B = 4096, 480, 60000
net = sdgc.gen_network(N, L, "radix")
bits = pack_rows(sdgc.gen_inputs(N, B)).view(np.int32)
g = SnicitNetwork.from_network(net)
st = torch.cuda.Stream()
g.set_stream(st)
src = {"device": torch.from_numpy(bits).cuda(), "pinned": torch.from_numpy(bits).pin_memory().numpy(), "pageable": bits}
for name in ("device", "pinned", "pageable", "device"):
    for pf in (1, 0):
        for _ in range(2):
            g.infer_packed(src[name], t=30, s=32, pre_fused=pf)
            g.categories()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(5):
            g.infer_packed(src[name], t=30, s=32, pre_fused=pf)
            c = g.categories()
        torch.cuda.synchronize()
        print(f"{name:9s} pre_fused={pf}: {(time.perf_counter() - t0) / 5 * 1e3:.3f} ms/step, {len(c)} categories", flush=True)
