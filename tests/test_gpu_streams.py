"""GPU: the library on user streams.  Kernels with dynamic tile queues
(fused-row / column-wise prefix, transpose) draw a queue slot per launch, and
every kernel is launched with programmatic dependent launch (griddepcontrol.wait
before any global access): launches in flight on several streams at once, and
chains of dependent launches with no host synchronisation in between, must give
exactly the results of one launch at a time."""
import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo

pytestmark = pytest.mark.gpu
DEV = "cuda"


def test_concurrent_streams_match_serial():
    n, p = 1024, 40000                       # the 128-instance TMA fused-row kernel, dynamic queue
    xs = [bo.generate_prefix(n, p, 20 + k, torch.float32, bo.ROW_WISE) for k in range(6)]
    ref = [bo.prefix_sums(x, bo.ROW_WISE) for x in xs]
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(3)]
    outs = [torch.empty_like(x) for x in xs]
    for rep in range(3):
        for k, x in enumerate(xs):
            s = streams[k % len(streams)]
            with torch.cuda.stream(s):
                bo.prefix_sums(x, bo.ROW_WISE, out=outs[k], stream=s)
        torch.cuda.synchronize()
        for k in range(len(xs)):
            assert torch.equal(outs[k].view(torch.int32), ref[k].view(torch.int32)), (rep, k)


def test_concurrent_triangulation_with_workspace():
    # TILED_GLOBAL keeps a table per CTA in the caller's workspace: one workspace per stream
    n, p = 80, 300
    cs = [bo.generate_tri(n, p, 30 + k, torch.float32, bo.ROW_WISE) for k in range(4)]
    ref = [bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL) for c in cs]
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(2)]
    need = bo.triangulation_workspace(n, p, bo.F32, bo.ROW_WISE, bo.TRI_TILED_GLOBAL)
    wss = [torch.empty(need, dtype=torch.uint8, device=DEV) for _ in streams]
    outs = [torch.empty(p, dtype=torch.float32, device=DEV) for _ in cs]
    for k, c in enumerate(cs):
        s = streams[k % 2]
        bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL, out=outs[k], workspace=wss[k % 2], stream=s)
    torch.cuda.synchronize()
    for k in range(len(cs)):
        assert torch.equal(outs[k].view(torch.int32), ref[k].view(torch.int32)), k


def test_dependent_chain_without_host_sync():
    # generate -> transpose -> column-wise prefix -> transpose back -> checksum, all queued on one
    # side stream with no synchronisation: each kernel reads what the previous one wrote
    n, p = 96, 5000
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        x = bo.generate_prefix(n, p, 41, torch.int32, bo.ROW_WISE, stream=s)
        xt = bo.transpose(x, stream=s)                                  # [n][p]
        bo.prefix_sums(xt, bo.COLUMN_WISE, out=xt, stream=s)           # in place
        y = bo.transpose(xt, stream=s)                                  # [p][n]
        z = bo.prefix_sums(y, bo.ROW_WISE, stream=s)                    # prefix of the prefix
    s.synchronize()
    h = bulkgen.prefix_input(n, p, seed=41, dtype="int32")
    once = oracle.bulk_prefix_sums(h, oracle.ROW_WISE)
    twice = oracle.bulk_prefix_sums(once, oracle.ROW_WISE)
    assert np.array_equal(y.cpu().numpy(), once)
    assert np.array_equal(z.cpu().numpy(), twice)


def test_cuda_graph_capture_and_replay():
    # the device entry points are capturable (launches with the PDL attribute become graph nodes,
    # tensor maps and queue slots are plain kernel arguments): tiny batches can skip the ~7 us of
    # host work per call by replaying a graph
    n, p = 32, 1024
    xs = [bo.generate_prefix(n, p, 50 + k, torch.int32, bo.ROW_WISE) for k in range(4)]
    c = bo.generate_tri(16, 512, 51, torch.int32, bo.ROW_WISE)
    ref_x = [bo.prefix_sums(x, bo.ROW_WISE) for x in xs]
    ref_c = bo.triangulation(c, bo.ROW_WISE)
    outs = [torch.empty_like(x) for x in xs]
    out_c = torch.empty_like(ref_c)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):                      # warm up on the capture stream
        for x, o in zip(xs, outs):
            bo.prefix_sums(x, bo.ROW_WISE, out=o, stream=s)
        bo.triangulation(c, bo.ROW_WISE, out=out_c, stream=s)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    for o in outs:
        o.zero_()
    out_c.zero_()
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        for x, o in zip(xs, outs):
            bo.prefix_sums(x, bo.ROW_WISE, out=o, stream=s)
        bo.triangulation(c, bo.ROW_WISE, out=out_c, stream=s)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    for o, r in zip(outs, ref_x):
        assert torch.equal(o, r)
    assert torch.equal(out_c, ref_c)


def test_graph_of_queue_kernels_beside_eager_launches():
    # the persistent fused-row / column-wise / transpose kernels claim tiles from a
    # device counter.  A captured launch takes no counter (static tile striding), eager launches
    # own one per stream, so replaying a graph of those kernels while eager launches of the same
    # kernels run on another stream can neither skip nor repeat a tile.
    n, p = 1024, 40000                                   # 128-instance fused-row kernel (dynamic queue)
    xs = [bo.generate_prefix(n, p, 60 + k, torch.float32, bo.ROW_WISE) for k in range(3)]
    xc = bo.generate_prefix(256, 40000, 64, torch.int32, bo.COLUMN_WISE)   # column-wise TMA ring
    ref = [bo.prefix_sums(x, bo.ROW_WISE) for x in xs]
    ref_c = bo.prefix_sums(xc, bo.COLUMN_WISE)
    ref_t = bo.transpose(xs[0])
    torch.cuda.synchronize()
    cap = torch.cuda.Stream()
    outs = [torch.empty_like(x) for x in xs]
    out_c = torch.empty_like(xc)
    out_t = torch.empty_like(ref_t)
    with torch.cuda.stream(cap):                          # warm-up on the capture stream
        for x, o in zip(xs, outs):
            bo.prefix_sums(x, bo.ROW_WISE, out=o, stream=cap)
    cap.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=cap):
        for x, o in zip(xs, outs):
            bo.prefix_sums(x, bo.ROW_WISE, out=o, stream=cap)
        bo.prefix_sums(xc, bo.COLUMN_WISE, out=out_c, stream=cap)
        bo.transpose(xs[0], out=out_t, stream=cap)
    eager = torch.cuda.Stream()
    e_outs = [torch.empty_like(x) for x in xs]
    for rep in range(4):
        for o in outs + e_outs:
            o.zero_()
        out_c.zero_()
        out_t.zero_()
        torch.cuda.synchronize()
        g.replay()                                       # on the current stream
        with torch.cuda.stream(eager):                   # overlapping eager launches, same kernels
            for x, o in zip(xs, e_outs):
                bo.prefix_sums(x, bo.ROW_WISE, out=o, stream=eager)
            bo.prefix_sums(xc, bo.COLUMN_WISE, stream=eager)
            bo.transpose(xs[0], stream=eager)
        torch.cuda.synchronize()
        for k in range(len(xs)):
            assert torch.equal(outs[k].view(torch.int32), ref[k].view(torch.int32)), (rep, k)
            assert torch.equal(e_outs[k].view(torch.int32), ref[k].view(torch.int32)), (rep, k)
        assert torch.equal(out_c, ref_c), rep
        assert torch.equal(out_t.view(torch.int32), ref_t.view(torch.int32)), rep


def test_out_tensor_is_validated():
    x = bo.generate_prefix(64, 100, 1, torch.float32, bo.ROW_WISE)
    with pytest.raises(ValueError):
        bo.prefix_sums(x, bo.ROW_WISE, out=torch.empty(64 * 99, dtype=torch.float32, device=DEV).view(99, 64))
    with pytest.raises(ValueError):
        bo.prefix_sums(x, bo.ROW_WISE, out=torch.empty_like(x, dtype=torch.int32))
    with pytest.raises(ValueError):
        bo.prefix_sums(x, bo.ROW_WISE, out=torch.empty(100, 64))           # host tensor
    c = bo.generate_tri(16, 50, 2, torch.int32, bo.ROW_WISE)
    with pytest.raises(ValueError):
        bo.triangulation(c, bo.ROW_WISE, out=torch.empty(49, dtype=torch.int32, device=DEV))
    with pytest.raises(ValueError):
        bo.triangulation(c, bo.ROW_WISE, out=torch.empty(50, dtype=torch.float32, device=DEV))


def test_captured_helper_replays_many_small_calls():
    # bo.Captured: a sequence of small bulk calls recorded once; replays give the eager results
    xs = [bo.generate_prefix(32, 1024, 70 + k, torch.int32, bo.ROW_WISE) for k in range(8)]
    c = bo.generate_tri(16, 256, 71, torch.int32, bo.ROW_WISE)
    ys = [torch.empty_like(x) for x in xs]
    oc = torch.empty(256, dtype=torch.int32, device=DEV)

    def step(s):
        for x, y in zip(xs, ys):
            bo.prefix_sums(x, bo.ROW_WISE, out=y, stream=s)
        bo.triangulation(c, bo.ROW_WISE, out=oc, stream=s)

    cap = bo.Captured(step)
    for y in ys:
        y.zero_()
    oc.zero_()
    torch.cuda.synchronize()
    for _ in range(3):
        cap.replay()
    torch.cuda.synchronize()
    for x, y in zip(xs, ys):
        assert torch.equal(y, bo.prefix_sums(x, bo.ROW_WISE))
    assert torch.equal(oc, bo.triangulation(c, bo.ROW_WISE))
