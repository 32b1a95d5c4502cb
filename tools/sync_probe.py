"""Isolated (host-synchronised) vs back-to-back launch timing per occupancy level.

The Fig. 9 tuner times one launch per explored level; this probe shows how far a launch
timed after a host sync is from the same level timed back to back (the steady state the
final kernel runs in).  Usage: python tools/sync_probe.py [hotspot2h_f32|srad_f32|nlm_f4]
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

kern = sys.argv[1] if len(sys.argv) > 1 else "hotspot2h_f32"
torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
if kern.startswith("hotspot") or kern.startswith("srad"):
    W = H = 8192
    a = torch.empty((H, W), device="cuda")
    p = torch.empty_like(a)
    b = torch.empty_like(a)
    O.generate_thermal(0, a.data_ptr(), p.data_ptr(), W, H, stream=sp)
    q0 = torch.full((1,), 3e-4, device="cuda")
    if kern.startswith("srad"):
        args = [O.srad_args(a.data_ptr(), b.data_ptr(), q0.data_ptr(), W, H),
                O.srad_args(b.data_ptr(), a.data_ptr(), q0.data_ptr(), W, H)]
    else:
        args = [O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H),
                O.hotspot_args(b.data_ptr(), a.data_ptr(), p.data_ptr(), W, H)]
else:
    W = H = 2048
    a = torch.empty((H, W, 4), device="cuda")
    b = torch.empty_like(a)
    O.generate_rgba(0, a.data_ptr(), W, H, stream=sp)
    args = [O.denoise_args(kern, a.data_ptr(), b.data_ptr(), W, H)] * 2
v, _ = O.build_all_levels(0, kern, mode=O.REALISE_MIN_CARVEOUT)
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(40)]
for i in range(len(v)):
    for _ in range(3):
        v.launch(i, args[0], sp)
    torch.cuda.synchronize()
    iso = []
    for r in range(15):
        e0, e1 = ev[r]
        e0.record()
        v.launch(i, args[r % 2], sp)
        e1.record()
        e1.synchronize()
        iso.append(e0.elapsed_time(e1))
    for r in range(40):
        e0, e1 = ev[r]
        e0.record()
        v.launch(i, args[r % 2], sp)
        e1.record()
    torch.cuda.synchronize()
    b2b = [e0.elapsed_time(e1) for e0, e1 in ev]
    print(f"k={v.level(i).ctas_per_sm:2d} cap={v.level(i).reg_cap:3d} isolated first={iso[0]:.4f} "
          f"median={statistics.median(iso):.4f} min={min(iso):.4f} | back-to-back median={statistics.median(b2b):.4f} "
          f"min={min(b2b):.4f}")
