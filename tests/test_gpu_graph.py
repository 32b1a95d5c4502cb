"""orion_tuner_capture / orion_graph_launch: once Fig. 9 has set the final kernel (PAPER.md
P:L643), n settled iterations replay as one CUDA graph -- bit-identical to launching them one
by one, counted as n launches, refused while the tuner is still exploring."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def knn():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return O.build_all_levels(0, "knn_f4", mode=O.REALISE_MIN_CARVEOUT)[0]


def test_graph_replay_matches_direct_launches(knn):
    W = H = 64
    n = 6
    sp = torch.cuda.current_stream().cuda_stream
    srcs = [torch.from_numpy(synth.noisy_rgba(W, H, seed=10 + f, sigma=0.2)).cuda() for f in range(n)]
    dsts = [torch.zeros_like(s) for s in srcs]
    args = [O.denoise_args("knn_f4", srcs[f].data_ptr(), dsts[f].data_ptr(), W, H) for f in range(n)]
    tuner = O.Tuner(knn)
    with pytest.raises(O.OrionError) as e:          # still exploring
        tuner.capture(args)
    assert e.value.status == -7
    it = 0
    while tuner.final()[0] < 0:
        tuner.step(args[it % n], sp)
        it += 1
        assert it < 200
    final = tuner.final()[0]
    ref = []
    for f in range(n):
        knn.launch(final, args[f], sp)
    torch.cuda.synchronize()
    ref = [d.cpu().numpy().copy() for d in dsts]
    for d in dsts:
        d.zero_()
    g = tuner.capture(args)
    c0 = O.launch_count()
    for _ in range(3):
        g.launch(sp)
    torch.cuda.synchronize()
    assert O.launch_count() - c0 == 3 * n
    for f in range(n):
        assert np.array_equal(dsts[f].cpu().numpy(), ref[f])
    g.close()


def test_resume_skips_exploration(knn):
    W = H = 64
    sp = torch.cuda.current_stream().cuda_stream
    src = torch.from_numpy(synth.noisy_rgba(W, H, seed=2, sigma=0.2)).cuda()
    dst = torch.zeros_like(src)
    a = O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), W, H)
    t = O.Tuner(knn)
    with pytest.raises(O.OrionError):
        t.resume(len(knn))
    t.resume(len(knn) - 1)
    r = t.step(a, sp)
    assert r.phase == 1 and r.level_idx == len(knn) - 1 and t.final()[0] == len(knn) - 1
    g = t.capture([a])                       # settled: capturable at once
    g.launch(sp)
    torch.cuda.synchronize()
    g.close()


def test_trace_jsonl(knn, tmp_path):
    import json
    W = H = 64
    sp = torch.cuda.current_stream().cuda_stream
    src = torch.from_numpy(synth.noisy_rgba(W, H, seed=4, sigma=0.2)).cuda()
    dst = torch.zeros_like(src)
    a = O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), W, H)
    path = tmp_path / "trace.jsonl"
    t = O.Tuner(knn, trace=str(path))
    for _ in range(12):
        t.step(a, sp)
    t.close()
    recs = [json.loads(line) for line in open(path)]
    assert [r["iteration"] for r in recs] == list(range(12))
    assert recs[0]["phase"] == "explore" and recs[0]["ms"] is not None
    assert all(r["ctas_per_sm"] >= 1 for r in recs)


def test_tune_steps_equals_step_loop(knn):
    # orion_tune_steps: n iterations in one library call == n orion_tune_step calls (same Fig. 9
    # walk, same final level, same output bits, n launches counted)
    W = H = 64
    n = 40
    sp = torch.cuda.current_stream().cuda_stream
    srcs = [torch.from_numpy(synth.noisy_rgba(W, H, seed=30 + f, sigma=0.2)).cuda() for f in range(4)]
    outs = []
    finals = []
    for mode in ("loop", "steps"):
        dsts = [torch.zeros_like(s) for s in srcs]
        args = [O.denoise_args("knn_f4", srcs[f % 4].data_ptr(), dsts[f % 4].data_ptr(), W, H) for f in range(n)]
        t = O.Tuner(knn)
        t.resume(len(knn) - 1)                      # a fixed final level: both runs launch the same kernel
        c0 = O.launch_count()
        if mode == "loop":
            for a in args:
                t.step(a, sp)
        else:
            r = t.steps(args, sp)
            assert r.final_level_idx == len(knn) - 1 and r.phase == 1
        torch.cuda.synchronize()
        assert O.launch_count() - c0 == n
        finals.append(t.final()[0])
        outs.append([d.cpu().numpy() for d in dsts])
    assert finals[0] == finals[1]
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


def test_graph_of_independent_frames_overlaps_and_matches(knn):
    # ORION_ARGS_INDEPENDENT frames captured with PDL on: the nodes keep programmatic edges and
    # skip griddepcontrol.wait (consecutive frames run concurrently); the bits are unchanged
    W = H = 64
    n = 24
    sp = torch.cuda.current_stream().cuda_stream
    prev = O.set_pdl(True)
    try:
        srcs = [torch.from_numpy(synth.noisy_rgba(W, H, seed=40 + f, sigma=0.2)).cuda() for f in range(n)]
        dsts = [torch.zeros_like(s) for s in srcs]
        args = [O.denoise_args("knn_f4", srcs[f].data_ptr(), dsts[f].data_ptr(), W, H, independent=True)
                for f in range(n)]
        tuner = O.Tuner(knn)
        it = 0
        while tuner.final()[0] < 0:
            tuner.step(args[it % n], sp)
            it += 1
            assert it < 200
        final = tuner.final()[0]
        refs = [torch.zeros_like(s) for s in srcs]
        for f in range(n):
            knn.launch(final, O.denoise_args("knn_f4", srcs[f].data_ptr(), refs[f].data_ptr(), W, H), sp)
        for d in dsts:
            d.zero_()
        g = tuner.capture(args)
        for _ in range(5):
            g.launch(sp)
        torch.cuda.synchronize()
        for f in range(n):
            assert torch.equal(dsts[f], refs[f]), f
        g.close()
        tuner.close()
    finally:
        O.set_pdl(prev)
