"""Small launches of every kernel family for compute-sanitizer (memcheck / racecheck /
synccheck; SURVEY §4 layer 3 and §5): C1-sized images, ragged edges, every level of each
kernel once, the SRAD statistics kernels (separate and fused), the generators, the fan-out
epilogue, row bands read from exactly-sized slabs, the hotspot / SRAD cp.async rings and
chained iterations (orion_chain).  Usage: compute-sanitizer --tool T python tools/sanitize_run.py"""
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
# row bands read from exactly-sized input slabs (a band height that is not a multiple of the tile
# height must not read past the slab: the C5 shard launch shape)
for k, halo in (("nlm_f4_w", 6), ("nlm_f4", 6), ("knn_f4", 3), ("knn_f4_t16", 3), ("nlm_f4_regheavy", 6)):
    v, _ = O.build_all_levels(0, k)
    r0, r1 = 10, 33
    s0, s1 = r0 - halo, r1 + halo
    slab = torch.empty((s1 - s0, W, 4), device="cuda")
    O.generate_rgba(0, slab.data_ptr(), W, H, s0, s1, sigma=0.13, stream=sp)
    band = torch.empty((r1 - r0, W, 4), device="cuda")
    v.launch(len(v) - 1, O.denoise_args(k, slab.data_ptr(), band.data_ptr(), W, H, r0, r1, s0, s1, r0), sp)
    torch.cuda.synchronize()
    print("ok band", k, flush=True)
WT, HT = 132, 37                                  # width % 4 == 0 for the float4 strips; srad takes any width
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
# SRAD with fused statistics: grids carry their statistics slots; the ROI spans two blocks
fa = torch.zeros(HT * 252 + O.SRAD_STATS_FLOATS, device="cuda")
fb = torch.zeros_like(fa)
O.generate_thermal(0, fa.data_ptr(), pw.data_ptr(), 252, HT, stream=sp)
roi = (2, 30, 100, 140)
O.srad_stats_init(0, fa.data_ptr(), 252, HT, roi, sp)
v, _ = O.build_all_levels(0, "srad_f32hs")
for i in (0, len(v) - 1):
    v.launch(i, O.srad_args(fa.data_ptr(), fb.data_ptr(), 0, 252, HT, roi=roi), sp)
    fa, fb = fb, fa
torch.cuda.synchronize()
print("ok srad_f32hs", flush=True)
# chained iterations (orion_chain: tile flags polled / published across launches), several tiles
# in both directions; every level once
WC, HC = 252, 1100
ca = torch.zeros(HC * WC + O.SRAD_STATS_FLOATS, device="cuda")
cb = torch.zeros_like(ca)
cp = torch.empty((HC, WC), device="cuda")
O.generate_thermal(0, ca.data_ptr(), cp.data_ptr(), WC, HC, stream=sp)
v, _ = O.build_all_levels(0, "hotspot4h_f32")
ch = O.Chain(v, WC, HC)
for i in list(range(len(v))) * 2:
    v.launch(i, O.hotspot_args(ca.data_ptr(), cb.data_ptr(), cp.data_ptr(), WC, HC, chain=ch), sp)
    ca, cb = cb, ca
torch.cuda.synchronize()
ch.close()
print("ok chained hotspot4h_f32", flush=True)
roi = (300, 700, 100, 200)
O.srad_stats_init(0, ca.data_ptr(), WC, HC, roi, sp)
v, _ = O.build_all_levels(0, "srad_f32hs")
ch = O.Chain(v, WC, HC)
for i in list(range(len(v))) * 2:
    v.launch(i, O.srad_args(ca.data_ptr(), cb.data_ptr(), 0, WC, HC, roi=roi, chain=ch), sp)
    ca, cb = cb, ca
torch.cuda.synchronize()
ch.close()
print("ok chained srad_f32hs", flush=True)
print("sanitize run complete")
