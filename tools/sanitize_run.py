"""Small launches of every kernel family for compute-sanitizer (memcheck / racecheck /
synccheck; SURVEY §4 layer 3 and §5): C1-sized images, ragged edges, every level of each
kernel once, the SRAD statistics kernel, the generators, the fan-out epilogue and the
hotspot / SRAD cp.async rings.  Usage: compute-sanitizer --tool T python tools/sanitize_run.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
W, H = 70, 45                                     # ragged: not a multiple of any tile
img = torch.empty((H, W, 4), device="cuda")
O.generate_rgba(0, img.data_ptr(), W, H, sigma=0.13, stream=sp)
for k in ("knn_f4", "knn_f4_p1", "knn_f4_t16", "nlm_f4", "nlm_f4_w", "nlm_f4_direct", "nlm_f4_regheavy"):
    v, _ = O.build_all_levels(0, k)
    out = torch.empty_like(img)
    full = torch.empty_like(img)
    for i in (0, len(v) - 1):
        a = O.denoise_args(k, img.data_ptr(), out.data_ptr(), W, H)
        if k in ("knn_f4", "knn_f4_p1", "knn_f4_t16", "nlm_f4", "nlm_f4_w"):
            a = O.with_fanout(a, [full.data_ptr()])
        v.launch(i, a, sp)
    torch.cuda.synchronize()
    print("ok", k, flush=True)
WT, HT = 132, 37                                  # width % 4 == 0 for hotspot2; srad takes any width
t0 = torch.empty((HT, WT), device="cuda")
pw = torch.empty_like(t0)
t1 = torch.empty_like(t0)
O.generate_thermal(0, t0.data_ptr(), pw.data_ptr(), WT, HT, stream=sp)
q0 = torch.empty(1, device="cuda")
for k in ("hotspot_f32", "hotspot2h_f32", "hotspot4h_f32", "srad_f32", "srad_f32h", "srad_f32_tile"):
    v, _ = O.build_all_levels(0, k)
    for w in ((WT, WT - 3) if k in ("srad_f32", "srad_f32_tile") else (WT,)):
        for i in (0, len(v) - 1):
            if k.startswith("srad"):
                O.srad_roi_stats(0, t0.data_ptr(), w, HT, (0, 20, 0, 20), q0.data_ptr(), sp)
                a = O.srad_args(t0.data_ptr(), t1.data_ptr(), q0.data_ptr(), w, HT)
            else:
                a = O.hotspot_args(t0.data_ptr(), t1.data_ptr(), pw.data_ptr(), w, HT)
            v.launch(i, a, sp)
    torch.cuda.synchronize()
    print("ok", k, flush=True)
print("sanitize run complete")
