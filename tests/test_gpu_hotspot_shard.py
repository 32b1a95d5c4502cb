"""The thermal stencil row-sharded with a halo exchange per launch ("the stencil (C3)
would need a halo exchange every step ... its sharded version is a NEXT item"): each band keeps
its rows plus 4 halo rows per side; a 4-step `hotspot4h_f32` launch on a band stores its first /
last 4 output rows straight into the neighbouring bands' next input buffers (orion_args.fanout =
the halo exchange), so after every launch each band's next input is complete.  Here the bands
are launched one after another on one GPU with plain buffers standing in for the peers' (the
same stores go over NVLink to symmetric-memory buffers in bench.py's multi-GPU C3); after 25
launches = 100 steps the union of the bands must equal the oracle's fp32 form bit for bit
(reading R-HS-S: the exchanged halo rows are exactly the cells a whole-grid launch would use)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402
from paper_conf_middleware_hayeslcsz16_b200 import shard  # noqa: E402

S = 4      # steps per launch = halo rows per side


@pytest.fixture(scope="module")
def v():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return O.build_all_levels(0, "hotspot4h_f32", mode=O.REALISE_MIN_CARVEOUT)[0]


def run_sharded(v, t0, pw, P, launches):
    H, W = t0.shape
    sp = torch.cuda.current_stream().cuda_stream
    bands = [shard.band(r, P, H, S) for r in range(P)]
    cur, nxt, pws = [], [], []
    for b in bands:
        cur.append(torch.from_numpy(np.ascontiguousarray(t0[b.src_begin:b.src_end])).cuda())
        nxt.append(torch.full((b.src_rows, W), float("nan"), device="cuda"))
        pws.append(torch.from_numpy(np.ascontiguousarray(pw[b.src_begin:b.src_end])).cuda())

    def gptr(t, b):          # global row y of band b's buffer t at gptr + y * W floats
        return t.data_ptr() - b.src_begin * W * 4

    for n in range(launches):
        for r, b in enumerate(bands):
            if not b.rows:
                continue
            a = O.hotspot_args(cur[r].data_ptr(), nxt[r].data_ptr(), pws[r].data_ptr(), W, H, b.row_begin,
                               b.row_end, src_row_begin=b.src_begin, src_row_end=b.src_end,
                               dst_row_begin=b.src_begin)
            up = gptr(nxt[r - 1], bands[r - 1]) if r > 0 else 0
            down = gptr(nxt[r + 1], bands[r + 1]) if r + 1 < P and bands[r + 1].rows else 0
            a = O.with_fanout(a, [up or None, down or None])
            v.launch((r + n) % len(v), a, sp)          # bands at different levels
        cur, nxt = nxt, cur
    torch.cuda.synchronize()
    out = np.empty((H, W), np.float32)
    for r, b in enumerate(bands):
        if b.rows:
            out[b.row_begin:b.row_end] = cur[r][b.row_begin - b.src_begin:b.row_end - b.src_begin].cpu().numpy()
    return out


@pytest.mark.parametrize("W,H,P", [(300, 203, 3), (256, 130, 2), (132, 61, 4), (300, 40, 5)])
def test_sharded_halo_exchange_equals_oracle(v, W, H, P):
    t0, pw = synth.thermal_inputs(W, H, seed=7)
    got = run_sharded(v, t0, pw, P, 25)
    assert np.array_equal(got, oracle.hotspot(t0, pw, 100, precision="f32"))


def test_sharded_equals_whole_grid_launches(v):
    W, H, P = 512, 300, 3
    t0, pw = synth.thermal_inputs(W, H, seed=8)
    got = run_sharded(v, t0, pw, P, 6)
    sp = torch.cuda.current_stream().cuda_stream
    a, b = torch.from_numpy(t0).cuda(), torch.empty((H, W), device="cuda")
    p = torch.from_numpy(pw).cuda()
    for _ in range(6):
        v.launch(len(v) - 1, O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H), sp)
        a, b = b, a
    torch.cuda.synchronize()
    assert np.array_equal(got, a.cpu().numpy())


def test_halo_fanout_argument_checks(v):
    sp = torch.cuda.current_stream().cuda_stream
    t = torch.empty((16, 64), device="cuda")
    a = O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), 64, 16)
    with pytest.raises(O.OrionError):
        v.launch(0, O.with_fanout(a, [t.data_ptr()]), sp)            # the exchange takes (upper, lower)


def test_symmetric_slabs_one_rank_nccl(v):
    # shard.SymmetricSlabs (the C3 multi-GPU slabs) on a one-rank NCCL group: a band launch whose
    # halo stores target the symmetric slabs' own addresses (as a neighbour's would over NVLink)
    # leaves the same bits as plain buffers
    import json
    import os
    import subprocess
    import sys
    code = r'''
import json, socket, torch, torch.distributed as dist
import numpy as np, synth
from paper_conf_middleware_hayeslcsz16_b200 import orion as O, shard
s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
torch.cuda.set_device(0)
dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", world_size=1, rank=0,
                        device_id=torch.device("cuda", 0))
W, H = 256, 96
t0, pw = synth.thermal_inputs(W, H, seed=3)
v, _ = O.build_all_levels(0, "hotspot4h_f32")
sl = shard.SymmetricSlabs(H, W, torch.device("cuda", 0))
sl.tensors[0].copy_(torch.from_numpy(t0))
p = torch.from_numpy(pw).cuda()
b = shard.band(0, 1, H, 4)
sp = torch.cuda.current_stream().cuda_stream
for n in range(5):
    cur, nxt = n % 2, (n + 1) % 2
    a = O.hotspot_args(sl.tensors[cur].data_ptr(), sl.tensors[nxt].data_ptr(), p.data_ptr(), W, H)
    # the halo stores of a band [0, H) land on the slab's own rows: a no-op by value
    a = O.with_fanout(a, [shard.global_row_ptr(sl.ptrs[nxt][0], b, W), shard.global_row_ptr(sl.ptrs[nxt][0], b, W)])
    v.launch(0, a, sp)
    sl.barrier()
torch.cuda.synchronize()
import oracle
print(json.dumps({"equal": bool(np.array_equal(sl.tensors[1].cpu().numpy(), oracle.hotspot(t0, pw, 20, precision="f32")))}))
dist.destroy_process_group()
'''
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600, cwd=root,
                       env=dict(os.environ, PYTHONPATH=root))
    assert r.returncode == 0, r.stderr[-3000:]
    assert json.loads(r.stdout.strip().splitlines()[-1]) == {"equal": True}
