"""GPU checks of the context's cached state across runs:
  * CUDA graphs captured by one run are never replayed after a later run reallocated a resident
    buffer they baked in (parameters alternating small -> large -> small on one registration);
  * output arrays bk_run page-locks are released at the end of the run unless the caller opted in
    (BK_FLAG_KEEP_OUTPUTS_PINNED), and released by bk_unpin_outputs then;
  * bk_run leaves the caller's current device unchanged;
  * the in/out struct size is validated for every kernel id, baseline flags included."""
import ctypes as C

import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu
MIB = 1 << 20


def is_registered(arr: np.ndarray) -> bool:
    """True iff `arr`'s memory is page-locked (cudaPointerGetAttributes type == cudaMemoryTypeHost),
    queried through the CUDA runtime torch already loaded (no error state left behind)."""
    import torch  # noqa: F401  (loads libcudart.so.12)

    class Attr(C.Structure):
        _fields_ = [("type", C.c_int), ("device", C.c_int), ("devicePointer", C.c_void_p), ("hostPointer", C.c_void_p)]

    rt = C.CDLL("libcudart.so.12")
    a = Attr()
    assert rt.cudaPointerGetAttributes(C.byref(a), C.c_void_p(arr.ctypes.data)) == 0
    return a.type == 1


@pytest.mark.parametrize("mode", ["dense", "zc"])
def test_groupby_alternating_G_replays_fresh_buffers(mode):
    n = 300_000
    g = gen.groupby(n=n, G=100)
    with bk.Context(window_bytes=2 * MIB, record_size=16, gather_mode=mode) as ctx:
        ctx.register(g, None, n_records=n)
        for G in (100, 8192, 100, 8192, 100):
            c, q, a = ctx.groupby(G)
            wc_, wq, wa = oracle.groupby(g, n, 16, G)
            assert np.array_equal(c, wc_) and np.array_equal(q, wq), G
            np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)


def test_grep_cap_small_large_small():
    gb, goff = gen.grep_records(n=40_000)
    want = oracle.grep(gb, goff, b"bigk")
    with bk.Context(window_bytes=1 * MIB, gather_mode="zc") as ctx:
        ctx.register(gb, goff)
        for cap in (len(want) + 1, len(goff), len(want) + 1, len(goff)):
            assert np.array_equal(ctx.grep(b"bigk", cap=cap), want), cap


def test_wordcount_kmer_wordcount_share_table():
    """word count and k-mers share the resident hash-table buffer: on one registration (256-B DNA
    read records, word count over whole fixed records), k-mers grow it between two word counts."""
    n = 6000
    d = gen.dna(n=n)
    want_wc = oracle.wc(d, np.arange(n, dtype=np.uint64) * 256)
    okm, oct_ = oracle.kmer(d, n, k=31)
    b = d.tobytes()
    for mode in ("zc", "auto"):   # the event pipeline, and the fused single launch over fixed records
        with bk.Context(window_bytes=1 * MIB, record_size=256, gather_mode=mode) as ctx:
            ctx.register(d, None, n_records=n)
            for step in range(3):
                o, l, c = ctx.wordcount(cap=1 << 17, table_slots=1 << 18)
                got = sorted((b[int(x): int(x) + int(y)], int(z)) for x, y, z in zip(o, l, c))
                assert got == want_wc, (mode, step)
                km, ct, _ = ctx.kmer(k=31, table_slots=1 << (20 + 2 * step), cap=1 << 20)
                o = np.argsort(km)
                assert np.array_equal(km[o], okm) and np.array_equal(ct[o], oct_), (mode, step)


def test_partition_buckets_alternate():
    n = 200_000
    kv = gen.kv(n=n)
    with bk.Context(window_bytes=2 * MIB, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
        for B in (256, 4096, 256):
            out, cc, bc = ctx.partition(B)
            assert np.array_equal(bk.partition_materialize(out, cc), oracle.partition(kv, B)[1]), B


def test_outputs_released_after_run_unless_kept():
    n = 100_000
    x = gen.points(n=n)
    mu = x[:64]
    cid = np.zeros(n, np.int32)
    with bk.Context(window_bytes=2 * MIB, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        ctx.kmeans(mu, cid=cid)
        assert not is_registered(cid)          # per-run registration released
    cid2 = np.zeros(n, np.int32)
    with bk.Context(window_bytes=2 * MIB, record_size=64, keep_outputs_pinned=True) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        ctx.kmeans(mu, cid=cid2)
        assert is_registered(cid2)             # cached across runs (opt-in)
        ctx.kmeans(mu, cid=cid2)
        ctx.unpin_outputs()
        assert not is_registered(cid2)
    assert np.array_equal(cid, cid2)


@pytest.mark.parametrize("keep", [False, True])
def test_outputs_reregistered_across_runs_never_replay_stale_graphs(keep):
    """A captured graph's D2H copies target the output registration of the run that captured it. Runs
    that re-register the same array (per-run pinning), arrays freed and reallocated at the same
    address (fresh k-means cid arrays), and kept registrations released by bk_unpin_outputs must
    never replay a graph bound to a released registration (gpurun_out/r02f1: partition run twice on
    one registration crashed inside the driver). Many repetitions: the failure was intermittent."""
    n = 120_000
    kv = gen.kv(n=n)
    _, wout = oracle.partition(kv, 256)
    x = gen.points(n=60_000)
    _, _, kchk, kcid = oracle.kmeans(x, x[:64], want_cid=True)
    out = np.empty_like(kv)
    # kept registrations require the caller to keep the arrays alive (bk.h): then only the arrays
    # unpinned by bk_unpin_outputs and pinned again change; per-run pinning also sees fresh arrays
    out2, cid_kept = np.empty_like(kv), np.empty(60_000, np.int32)
    with bk.Context(window_bytes=1 * MIB, record_size=16, keep_outputs_pinned=keep) as pctx, \
            bk.Context(window_bytes=1 * MIB, record_size=64, keep_outputs_pinned=keep) as kctx:
        pctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
        kctx.register(x.view(np.uint8).reshape(-1), None, n_records=60_000)
        for it in range(12):
            out[:] = 0
            o, cc, _ = pctx.partition(256, out=out)
            assert np.array_equal(bk.partition_materialize(o, cc), wout), it
            fresh = out2 if keep else np.empty_like(kv)   # a new array, often at a recycled address
            o2, cc2, _ = pctx.partition(256, out=fresh)
            assert np.array_equal(bk.partition_materialize(o2, cc2), wout), it
            del fresh, o2
            cid = cid_kept if keep else np.empty(60_000, np.int32)
            cid[:] = -1
            _, _, chk = kctx.kmeans(x[:64], cid=cid)
            assert chk == kchk and np.array_equal(cid, kcid), it
            del cid
            if keep and it % 3 == 2:
                pctx.unpin_outputs()
                kctx.unpin_outputs()


def test_graph_issue_reported():
    """bk_stats.graph_issue: static pipelines capture a graph on the first run and replay it later
    (kept-pinned or no per-record outputs); outputs page-locked for one run only, NO_GRAPH and
    host-assembled (HYBRID) runs issue eagerly."""
    n = 100_000
    kv = gen.kv(n=n)
    out = np.empty_like(kv)
    g = gen.groupby(n=n)
    for keep, want in ((True, [1, 2, 2]), (False, [0, 0, 0])):
        with bk.Context(window_bytes=1 * MIB, record_size=16, keep_outputs_pinned=keep) as ctx:
            ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
            got = []
            for _ in range(3):
                ctx.partition(256, out=out)
                got.append(ctx.stats()["graph_issue"])
            assert got == want, (keep, got)
    for flags, want in (({}, [1, 2]), ({"no_graph": True}, [0, 0])):
        with bk.Context(window_bytes=1 * MIB, record_size=16, **flags) as ctx:
            ctx.register(g, None, n_records=n)
            got = []
            for _ in range(2):
                ctx.groupby(4096)
                got.append(ctx.stats()["graph_issue"])
            assert got == want, (flags, got)
    g64 = gen.groupby(n=n, stride=64)
    with bk.Context(window_bytes=1 * MIB, record_size=64, gather_mode="hybrid") as ctx:
        ctx.register(g64, None, n_records=n)
        ctx.groupby(4096)
        ctx.groupby(4096)
        assert ctx.stats()["graph_issue"] == 0


def test_current_device_restored_and_struct_size_checked():
    import torch
    torch.cuda.set_device(0)
    n = 10_000
    g = gen.groupby(n=n)
    for flags in ({}, {"baseline_dbuf": True}):
        with bk.Context(window_bytes=1 * MIB, record_size=16, **flags) as ctx:
            ctx.register(g, None, n_records=n)
            ctx.groupby(4096)
            assert torch.cuda.current_device() == 0
            o = bk._hdr(bk.bk_out_groupby, bk.BK_K_GROUPBY)
            o.h.struct_size = C.sizeof(bk.bk_out_grep)   # wrong size for this kernel id
            cnt = np.empty(4096, np.uint64)
            o.G, o.count, o.qty, o.amount = 4096, cnt.ctypes.data, cnt.ctypes.data, cnt.ctypes.data
            with pytest.raises(bk.BkError) as e:
                bk.bk_run(ctx.ctx, bk.BK_K_GROUPBY, None, o)
            assert e.value.status == bk.BK_E_INVAL


@pytest.mark.parametrize("mode", ["dense", "zc", "hybrid"])
def test_trace_flag_keeps_graph_replay_and_reports_stages(mode):
    """BK_FLAG_TRACE (CUPTI activity records) on the graph-replayed pipeline: results unchanged, the
    traced span is the run's device time, transfer and compute intervals are reported."""
    n = 400_000
    g = gen.groupby(n=n, stride=64)
    want = oracle.groupby(g, n, 64, 4096)
    with bk.Context(window_bytes=4 * MIB, record_size=64, gather_mode=mode, trace=True) as ctx:
        ctx.register(g, None, n_records=n)
        for _ in range(3):
            c, q, a = ctx.groupby(4096)
            assert np.array_equal(c, want[0]) and np.array_equal(q, want[1])
        st = ctx.stats()
    assert st["n_trace_records"] > st["n_chunks"] and st["ms_trace_span"] > 0
    assert st["ms_xfer_busy"] > 0 and st["ms_compute_busy"] > 0
    assert st["ms_trace_span"] <= st["ms_device"] * 1.05 + 0.05
