"""Time one kernel's launch (events, median of N back-to-back launches) over a list of frame
heights: how the time per tile behaves across the wave quantisation of the grid.

usage: python tools/wave_probe.py KERNEL LEVEL W H1 [H2 ...]
"""
import os
import sys
import statistics

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

kernel, lev, W = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
heights = [int(h) for h in sys.argv[4:]]
torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
v, res = O.build_all_levels(0, kernel, 0, mode=O.REALISE_MIN_CARVEOUT)
li = lev % len(v)
Hm = max(heights)
a = torch.empty((Hm, W, 4), device="cuda")
b = torch.empty((Hm, W, 4), device="cuda")
O.generate_rgba(0, a.data_ptr(), W, Hm, sigma=0.13, stream=sp)
for H in heights:
    args = O.denoise_args(kernel, a.data_ptr(), b.data_ptr(), W, H)
    for _ in range(5):
        v.launch(li, args, sp)
    ts = []
    for _ in range(30):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        v.launch(li, args, sp)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{kernel} level {li} W {W} H {H}: {statistics.median(ts):.4f} ms  {W * H / statistics.median(ts) / 1e6:.2f} Gpix/s", flush=True)
