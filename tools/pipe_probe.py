"""Measure the host pipe at depths 1..4 and raw pinned H2D / D2H copy bandwidth (C2 frames)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

W = H = 2048
torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
src = torch.empty((H, W, 4), device="cuda")
O.generate_rgba(0, src.data_ptr(), W, H, stream=sp)
hin = [src.cpu().pin_memory() for _ in range(4)]
hout = [torch.empty((H, W, 4)).pin_memory() for _ in range(4)]
d = torch.empty_like(src)
torch.cuda.synchronize()
for name, fn in (("h2d", lambda: d.copy_(hin[0], non_blocking=True)), ("d2h", lambda: hout[0].copy_(d, non_blocking=True))):
    fn(); torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(20):
        fn()
    torch.cuda.synchronize()
    print(name, "GB/s", 20 * W * H * 16 / (time.perf_counter() - t) / 1e9)
s2 = torch.cuda.Stream()
t = time.perf_counter()
for _ in range(20):
    d.copy_(hin[0], non_blocking=True)
    with torch.cuda.stream(s2):
        hout[1].copy_(src, non_blocking=True)
torch.cuda.synchronize()
print("h2d+d2h concurrent GB/s each", 20 * W * H * 16 / (time.perf_counter() - t) / 1e9)
v, _ = O.build_all_levels(0, "nlm_f4")
t_ = O.Tuner(v)
for depth in (1, 2, 3, 4):
    pipe = O.HostPipe(t_, W, H, depth=depth)
    args = [O.denoise_args("nlm_f4", hin[f].data_ptr(), hout[f].data_ptr(), W, H) for f in range(4)]
    for f in range(depth):
        pipe.submit(args[f])
    pipe.drain()
    n = 40
    t0 = time.perf_counter()
    for s in range(n):
        pipe.submit(args[s % 4])
    pipe.drain()
    dt = time.perf_counter() - t0
    print("depth", depth, "Mpix/s", n * W * H / dt / 1e6, "ms/frame", dt / n * 1e3)
    pipe.close()
