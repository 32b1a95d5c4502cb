"""Bit-identity of two liborion builds on the SRAD kernels (run on a gpurun box).

    python tools/lib_bitcmp.py build/liborion_A.so paper_conf_middleware_hayeslcsz16_b200/liborion.so

Each library runs in its own subprocess (ORION_LIB), every SRAD kernel id at every level on a
seeded 1000x1000 grid for 20 iterations (and the 4096^2 bench grid for 4); the outputs are hashed
and the two libraries' hashes compared.  Prints one JSON line {"identical": bool, ...}.
"""
import hashlib
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import hashlib, json, numpy as np, torch, synth
from paper_conf_middleware_hayeslcsz16_b200 import orion as O
sp = torch.cuda.current_stream().cuda_stream
out = {}
for kernel in ["srad_f32", "srad_f32h", "srad_f32_tile", "srad_f32hs"]:
    v, _ = O.build_all_levels(0, kernel, mode=O.REALISE_MIN_CARVEOUT)
    for (W, H, iters) in [(1000, 1000, 20), (4096, 4096, 4)]:
        j0, _ = synth.thermal_inputs(W, H, seed=11)
        roi = (0, min(H, 256) - 1, 0, min(W, 256) - 1)   # <= 64 statistics slots
        for lvl in range(len(v)):
            n = H * W + O.SRAD_STATS_FLOATS
            a = torch.zeros(n, device="cuda"); b = torch.zeros(n, device="cuda")
            a[:H * W] = torch.from_numpy(np.ascontiguousarray(j0, dtype=np.float32).ravel()).cuda()
            q0 = torch.empty(1, device="cuda")
            if kernel == "srad_f32hs":
                O.srad_stats_init(0, a.data_ptr(), W, H, roi, sp)
            for _ in range(iters):
                if kernel == "srad_f32hs":
                    v.launch(lvl, O.srad_args(a.data_ptr(), b.data_ptr(), 0, W, H, 0.5, roi=roi), sp)
                else:
                    O.srad_roi_stats(0, a.data_ptr(), W, H, roi, q0.data_ptr(), sp)
                    v.launch(lvl, O.srad_args(a.data_ptr(), b.data_ptr(), q0.data_ptr(), W, H, 0.5), sp)
                a, b = b, a
            torch.cuda.synchronize()
            out[f"{kernel}/{W}x{H}/L{lvl}"] = hashlib.sha256(a[:H * W].cpu().numpy().tobytes()).hexdigest()[:16]
    v.close()
print(json.dumps(out))
'''


def run(lib):
    r = subprocess.run([sys.executable, "-c", CHILD], capture_output=True, text=True, cwd=ROOT,
                       env=dict(os.environ, ORION_LIB=lib, PYTHONPATH=ROOT), timeout=900)
    if r.returncode:
        sys.exit(r.stderr[-3000:])
    return json.loads(r.stdout.strip().splitlines()[-1])


def main():
    a, b = run(sys.argv[1]), run(sys.argv[2])
    diff = sorted(k for k in a if a[k] != b.get(k))
    print(json.dumps({"identical": not diff and a.keys() == b.keys(), "cases": len(a), "differ": diff}))


if __name__ == "__main__":
    main()
