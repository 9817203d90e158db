"""The asynchronous entry points (vs_run_async, vs_score_poses_device) with arbitrary caller streams.

Both run on the ctx's own stream joined to the caller's stream by events (include/vs.h), so:
  * repeated vs_run_async calls on the legacy default stream (stream=None in the binding is torch's current
    stream, the legacy NULL stream by default) replay a CUDA graph captured on the ctx stream;
  * a vs_score_poses_device and a vs_run_async of one ctx on two different caller streams never overlap
    (they share the ctx's scratch buffers), and each result equals the synchronous call's bit for bit.
"""
import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import synth, vs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def test_run_async_repeated_on_legacy_stream(torch):
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    mp = vs.mh_preset(3, population=32, generations=3)
    ns = prob.cfg.n_spots
    ref = {s: g.run(mp, s) for s in (1, 2, 3)}
    g2 = vs.Context.from_problem(prob, vs.score_params())
    bp = torch.empty((ns, 7), device="cuda")
    bs = torch.empty(ns, device="cuda")
    assert torch.cuda.current_stream().cuda_stream == 0          # the legacy default stream
    for seed in (1, 2, 3, 1, 2):                                   # 2nd identical call captures, later ones replay
        g2.run_async(mp, seed, None, bp, bs)                      # stream=None -> current (legacy) stream
        np.testing.assert_array_equal(bs.cpu().numpy(), ref[seed][1])
        np.testing.assert_array_equal(bp.cpu().numpy(), ref[seed][0])


def test_async_calls_on_two_streams_do_not_overlap(torch):
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    ns = prob.cfg.n_spots
    mp = vs.mh_preset(3, population=64, generations=4)
    pref, sref = g.run(mp, 5)
    spot, q, t = synth.make_poses(20000, ns, 3.0, seed=3)
    href = g.score_poses(spot, q, t)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    sd, qd, td = (torch.from_numpy(x).cuda() for x in (spot, q, t))
    out = torch.empty(len(spot), device="cuda")
    bp = torch.empty((ns, 7), device="cuda")
    bs = torch.empty(ns, device="cuda")
    torch.cuda.synchronize()
    for rep in range(3):
        out.zero_()
        bs.zero_()
        with torch.cuda.stream(s1):
            g.score_poses_device(sd, qd, td, out, s1)
        with torch.cuda.stream(s2):
            g.run_async(mp, 5, None, bp, bs, s2)
        s1.synchronize()
        s2.synchronize()
        np.testing.assert_array_equal(out.cpu().numpy(), href)
        np.testing.assert_array_equal(bs.cpu().numpy(), sref)
        np.testing.assert_array_equal(bp.cpu().numpy(), pref)


def test_caller_stream_ordering(torch):
    """Work enqueued on the caller's stream before the call is visible to it; work after it sees its results."""
    prob = synth.make_problem("tiny")
    g = vs.Context.from_problem(prob, vs.score_params())
    spot, q, t = synth.make_poses(4096, prob.cfg.n_spots, 3.0, seed=9)
    href = g.score_poses(spot, q, t)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        torch.cuda._sleep(20_000_000)                             # delay the caller's stream (~10 ms)
        qd = torch.from_numpy(q).cuda(non_blocking=False)
        sd = torch.from_numpy(spot).cuda()
        td = torch.from_numpy(t).cuda()
        out = torch.full((len(spot),), float("nan"), device="cuda")
        g.score_poses_device(sd, qd, td, out, st)
        res = out * 1.0                                           # consumer on the caller's stream
    st.synchronize()
    np.testing.assert_array_equal(res.cpu().numpy(), href)
