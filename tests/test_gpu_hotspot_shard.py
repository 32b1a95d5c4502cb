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
