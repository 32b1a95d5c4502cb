import sys, time
sys.path.insert(0, '.')
from paper_conf_middleware_hayeslcsz16_b200 import orion as O
for k in ["srad_f32", "hotspot_f32", "hotspot2_f32", "knn_f4", "nlm_f4_regheavy", "nlm_f4"]:
    for mode in (O.REALISE_MIN_CARVEOUT, O.REALISE_MAX_SMEM):
        t = time.time()
        v, res = O.build_all_levels(0, k, mode=mode)
        print(k, "min" if mode else "max", f"{time.time()-t:.2f}s", [(v.level(i).ctas_per_sm, v.level(i).smem_pad_bytes, v.level(i).carveout_kb, v.planned[i].carveout_kb, v.info(i).verified_ctas) for i in range(len(v))])
