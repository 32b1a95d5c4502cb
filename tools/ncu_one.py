"""Launch ONE kernel variant once on a synthetic frame (for ncu --set full captures).

usage: python tools/ncu_one.py KERNEL LEVEL W H [THREADS] [REPEAT] [BATCH]
  LEVEL = index into the level list (-1 = max occupancy, 'orig' = natural build, 'best' = the
  sweep's fastest level, 'all' = every level once, in order).  Levels are realised as bench.py realises them (MIN_CARVEOUT).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

kernel, lev, W, H = sys.argv[1], sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
threads = int(sys.argv[5]) if len(sys.argv) > 5 else 0
repeat = int(sys.argv[6]) if len(sys.argv) > 6 else 1
batch = int(sys.argv[7]) if len(sys.argv) > 7 else 1     # frames per launch (orion_args.batch)
torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
mode = O.REALISE_MAX_SMEM if os.environ.get("ORION_REALISE") == "max" else O.REALISE_MIN_CARVEOUT
v, res = O.build_all_levels(0, kernel, threads, mode=mode)
if lev in ("all", "best"):
    li = None
elif lev == "orig":
    li = max((i for i, l in enumerate(v.planned) if l.reg_cap == 0), key=lambda i: v.planned[i].ctas_per_sm)
else:
    li = int(lev) % len(v)
if kernel.startswith("srad"):
    extra = O.SRAD_STATS_FLOATS if kernel == "srad_f32hs" else 0
    a = torch.empty(H * W + extra, device="cuda")
    b = torch.empty(H * W + extra, device="cuda")
    p = torch.empty((H, W), device="cuda")
    q0 = torch.empty(1, device="cuda")
    O.generate_thermal(0, a.data_ptr(), p.data_ptr(), W, H, stream=sp)
    if extra:
        O.srad_stats_init(0, a.data_ptr(), W, H, (0, 127, 0, 127), sp)
        args = O.srad_args(a.data_ptr(), b.data_ptr(), 0, W, H, roi=(0, 127, 0, 127))
    else:
        O.srad_roi_stats(0, a.data_ptr(), W, H, (0, 127, 0, 127), q0.data_ptr(), sp)
        args = O.srad_args(a.data_ptr(), b.data_ptr(), q0.data_ptr(), W, H)
elif kernel.startswith("hotspot"):
    a = torch.empty((H, W), device="cuda")
    b = torch.empty((H, W), device="cuda")
    p = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, a.data_ptr(), p.data_ptr(), W, H, stream=sp)
    args = O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H)
else:
    a = torch.empty((batch, H, W, 4), device="cuda")
    b = torch.empty((batch, H, W, 4), device="cuda")
    for f in range(batch):
        O.generate_rgba(0, a[f].data_ptr(), W, H, seed=1 + f, sigma=0.13, stream=sp)
    args = O.denoise_args(kernel, a.data_ptr(), b.data_ptr(), W, H, batch=batch)
torch.cuda.synchronize()
if lev == "best":   # the exhaustive sweep's fastest level (what the tuner should settle on)
    ms = v.sweep(args, sp, rounds=5)
    li = min(range(len(ms)), key=lambda i: ms[i])
torch.cuda.nvtx.range_push("measure")   # ncu --nvtx --nvtx-include "measure/": skips the build's probe launches
for i in (range(len(v)) if li is None else [li]):
    for _ in range(repeat):
        v.launch(i, args, sp)
    torch.cuda.synchronize()
    print("launched", kernel, "level", i, v.level(i), v.info(i))
torch.cuda.nvtx.range_pop()
