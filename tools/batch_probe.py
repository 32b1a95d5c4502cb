"""C1 with batched launches: every KNN kernel's sweep (every level) over batches of B 64x64
frames; prints ms per batch and us per frame at the best level.  Usage: python tools/batch_probe.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

torch.cuda.set_device(0)
sp = torch.cuda.current_stream().cuda_stream
W = H = 64
for B in (16, 64, 256):
    src = torch.empty((B, H, W, 4), device="cuda")
    for f in range(B):
        O.generate_rgba(0, src[f].data_ptr(), W, H, seed=1 + f, sigma=0.2, stream=sp)
    dst = torch.empty_like(src)
    for k in ("knn_f4_t16", "knn_f4", "knn_f4_p1"):
        for T in ((128,) if k != "knn_f4" else (128, 256, 64)):
            v, _ = O.build_all_levels(0, k, block_threads=T, mode=O.REALISE_MIN_CARVEOUT)
            ms = v.sweep(O.denoise_args(k, src.data_ptr(), dst.data_ptr(), W, H, batch=B), sp, rounds=5)
            i = min(range(len(v)), key=lambda j: ms[j])
            print(f"B={B} {k} T={T} best k={v.level(i).ctas_per_sm} {ms[i]:.4f} ms/batch = {1e3 * ms[i] / B:.3f} us/frame;"
                  f" levels {[round(m, 4) for m in ms]}", flush=True)
            v.close()
