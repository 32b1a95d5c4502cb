"""Print every kernel's realised levels in both realisation modes:
(k, pad bytes, realised carveout KB, planned carveout KB, MEASURED CTAs/SM) per level, and the
build time (ptxas per register cap + one residency probe per candidate configuration)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

kernels = sys.argv[1:] or ["srad_f32", "hotspot_f32", "hotspot2h_f32", "knn_f4", "nlm_f4_regheavy", "nlm_f4"]
for k in kernels:
    for mode in (O.REALISE_MIN_CARVEOUT, O.REALISE_MAX_SMEM):
        t = time.time()
        v, res = O.build_all_levels(0, k, mode=mode)
        print(k, "min_carveout" if mode else "max_smem", f"{time.time() - t:.2f}s",
              [(v.level(i).ctas_per_sm, v.level(i).smem_pad_bytes, v.level(i).carveout_kb, v.planned[i].carveout_kb,
                v.info(i).verified_ctas) for i in range(len(v))])
