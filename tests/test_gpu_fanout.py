"""Fan-out epilogue (orion_args.fanout): a row-sharded frame gathered by the kernels' own
stores into every rank's full image (C5 without a separate all-gather).  Here the "ranks" are
row bands launched on one GPU and the fan-out buffers are plain device buffers -- the same
stores a peer pointer receives over NVLink.  Results must equal the unsharded launch bit for
bit in every buffer."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402
from paper_conf_middleware_hayeslcsz16_b200 import shard  # noqa: E402


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


@pytest.mark.parametrize("kernel,halo", [("nlm_f4", 6), ("knn_f4", 3), ("knn_f4_t16", 3), ("nlm_f4_w", 6)])
@pytest.mark.parametrize("P", [2, 3])
def test_fanout_gathers_bands_bit_exact(dev, kernel, halo, P):
    W, H = 250, 131
    sp = torch.cuda.current_stream().cuda_stream
    v, _ = O.build_all_levels(0, kernel)
    img = torch.from_numpy(synth.noisy_rgba(W, H, seed=3, sigma=0.13)).cuda()
    full_ref = torch.empty_like(img)
    v.launch(len(v) - 1, O.denoise_args(kernel, img.data_ptr(), full_ref.data_ptr(), W, H), sp)
    fulls = [torch.full_like(img, -1.0) for _ in range(P)]
    for r in range(P):
        b = shard.band(r, P, H, halo)
        if not b.rows:
            continue
        slab = img[b.src_begin:b.src_end].contiguous()
        band = torch.empty((b.rows, W, 4), device="cuda")
        a = O.denoise_args(kernel, slab.data_ptr(), band.data_ptr(), W, H, b.row_begin, b.row_end, b.src_begin,
                           b.src_end, b.row_begin)
        v.launch(r % len(v), O.with_fanout(a, [f.data_ptr() for f in fulls]), sp)
        torch.cuda.synchronize()
        assert torch.equal(band, full_ref[b.row_begin:b.row_end])
    torch.cuda.synchronize()
    for f in fulls:
        assert torch.equal(f, full_ref)


def test_fanout_rejected_where_unsupported(dev):
    v, _ = O.build_all_levels(0, "hotspot_f32")
    t = torch.zeros((16, 128), device="cuda")
    a = O.with_fanout(O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), 128, 16), [t.data_ptr()])
    with pytest.raises(O.OrionError) as e:
        v.launch(0, a)
    assert e.value.status == -1


def test_symmetric_memory_fanout_one_rank_nccl(dev):
    # the C5 exchange as bench.py runs it over NCCL: the full image in torch symmetric memory
    # (shard.FanoutImage), the kernel's epilogue storing every band into it, the device barrier
    # closing the step -- here on a one-rank NCCL group (P > 1 needs more GPUs than gpurun has).
    # The bands are launched at different levels; the image equals the unsharded launch bit for bit.
    import json
    import os
    import subprocess
    import sys
    code = r'''
import json, socket, torch, torch.distributed as dist
from paper_conf_middleware_hayeslcsz16_b200 import orion as O, shard
s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
torch.cuda.set_device(0)
dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", world_size=1, rank=0,
                        device_id=torch.device("cuda", 0))
W, H, P = 700, 333, 3
sp = torch.cuda.current_stream().cuda_stream
v, _ = O.build_all_levels(0, "nlm_f4_w")
full_in = torch.empty((H, W, 4), device="cuda")
O.generate_rgba(0, full_in.data_ptr(), W, H, seed=3, sigma=0.13, stream=sp)
ref = torch.empty((H, W, 4), device="cuda")
v.launch(len(v) - 1, O.denoise_args("nlm_f4_w", full_in.data_ptr(), ref.data_ptr(), W, H), sp)
fan = shard.FanoutImage((H, W, 4), torch.device("cuda", 0))
for r in range(P):
    b = shard.band(r, P, H, 6)
    slab = torch.empty((b.src_rows, W, 4), device="cuda")
    O.generate_rgba(0, slab.data_ptr(), W, H, b.src_begin, b.src_end, seed=3, sigma=0.13, stream=sp)
    out = torch.empty((b.rows, W, 4), device="cuda")
    a = O.denoise_args("nlm_f4_w", slab.data_ptr(), out.data_ptr(), W, H, b.row_begin, b.row_end, b.src_begin,
                       b.src_end, b.row_begin)
    v.launch(r % len(v), O.with_fanout(a, fan.ptrs), sp)
fan.barrier()
torch.cuda.synchronize()
print(json.dumps({"equal": bool(torch.equal(fan.tensor, ref)), "nptrs": len(fan.ptrs)}))
dist.destroy_process_group()
'''
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600, cwd=root,
                       env=dict(os.environ, PYTHONPATH=root))
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d == {"equal": True, "nptrs": 1}


def test_bench_c5_fanout_path_one_gpu(dev):
    # bench.py's C5 measurement with the fan-out exchange requested on one GPU: the JSON line
    # names the symmetric-memory fan-out and reports compute, exchange and end-to-end figures
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--workload", "c5", "--only", "--size", "2048",
                        "--c5-mode", "fanout", "--steps", "3", "--warmup", "3", "--rounds", "3"],
                       capture_output=True, text=True, timeout=900, cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    assert "fan-out" in d["config"]["collective"] and d["n_gpus"] == 1
    assert d["value"] > 0 and d["compute_only"]["value"] > 0 and d["e2e"]["value"] > 0
    assert d["per_rank"][0]["final_k"] >= 1


def test_bench_c5_gather_path_one_gpu(dev):
    # bench.py's C5 with the chunked NCCL all-gather requested on one GPU (a one-rank NCCL group):
    # row chunks computed as kernel-split iterations, each chunk's all-gather on a side stream
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--workload", "c5", "--only", "--size", "2048",
                        "--c5-mode", "gather", "--steps", "3", "--warmup", "3", "--rounds", "3"],
                       capture_output=True, text=True, timeout=900, cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    assert "all_gather" in d["config"]["collective"] and d["n_gpus"] == 1, d["config"]
    assert d["value"] > 0 and d["compute_only"]["value"] > 0 and d["e2e"]["value"] > 0
