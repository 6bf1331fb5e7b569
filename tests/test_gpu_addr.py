"""Address mode (BK_GATHER_ADDR): the paper's own stages 1-3 with the online
pattern recogniser of §IV.A driving them. Every lane's element addresses are generated
on the GPU, compressed to base + strides where a pattern holds (else sent explicitly), assembled on
the host from exactly that information and DMA'd. Checked against the oracle:
  * the staged bytes of a chunk equal the layout oracle O-L, with and without patterns;
  * every built-in kernel's result equals the oracle in address mode, with and without patterns;
  * the address accounting matches the access spec (I3: every accessed byte once; explicit = all);
  * a caller's own address generator (bk_run_user_addr) drives stages 2-3 for its own stage 4."""
import ctypes as C
import os

import numpy as np
import pytest
import torch

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MIB = 1 << 20
M64 = (1 << 64) - 1


def wc_multiset_gpu(buf, off_, ln, cnt):
    b = buf.tobytes()
    return sorted((b[int(o): int(o) + int(l)], int(c)) for o, l, c in zip(off_, ln, cnt))


LAYOUT_CASES = [
    ("wc_text", None, 0),
    ("grep_key", [(16, 32)], 0),
    ("sparse64", [(0, 16)], 64),
    ("kmeans64", None, 64),
    ("dup_extents", [(8, 4), (0, 12), (8, 4)], 16),
    ("grep_multi", [(16, 8), (40, 8)], 0),
]


def layout_data(name):
    if name == "wc_text":
        buf, off = gen.text(cap_bytes=200_000)
        return buf, off, 0
    if name in ("grep_key", "grep_multi"):
        buf, off = gen.grep_records(n=4000)
        return buf, off, 0
    if name == "sparse64":
        return gen.groupby(n=7001, stride=64), None, 64
    if name == "kmeans64":
        return gen.points(n=3001).view(np.uint8).reshape(-1), None, 64
    return gen.groupby(n=4099, stride=16), None, 16


@pytest.mark.parametrize("name,extents,rs", LAYOUT_CASES)
@pytest.mark.parametrize("patterns", [True, False])
def test_addr_layout_matches_oracle(name, extents, rs, patterns):
    buf, off, rs = layout_data(name)
    n = len(off) if off is not None else len(buf) // rs
    with bk.Context(window_bytes=8 * MIB, n_slots=2, gather_mode="addr", chunk_bytes=12_000, lanes=64,
                    record_size=rs, no_patterns=not patterns) as ctx:
        ctx.register(buf, off, n_records=n)
        d0 = ctx.layout_dump(0, extents=extents)
        for c in sorted({0, 1, d0["n_chunks"] // 2, d0["n_chunks"] - 1}):
            d = ctx.layout_dump(c, extents=extents)
            stage, lf, ln, lb = oracle.layout(buf, off, n, len(buf), rs, extents, d["lo"], d["hi"], d["lanes"])
            assert np.array_equal(d["lane_first"], lf) and np.array_equal(d["lane_nrec"], ln)
            assert np.array_equal(d["lane_bytes"], lb)
            assert d["stage"].tobytes() == stage.tobytes(), (name, c)
        st = ctx.stats()
    assert st["gather_mode"] == bk.BK_GATHER_ADDR and st["n_addr_lanes"] > 0
    if not patterns:
        assert st["n_pattern_lanes"] == 0 and st["n_explicit_addr"] == st["n_addresses"]


def test_addr_all_kernels_match_oracle():
    for patterns in (True, False):
        kw = dict(gather_mode="addr", no_patterns=not patterns)
        # word count (1-B elements: the paper's "an address for each accessed character")
        buf, off = gen.text(cap_bytes=1 * MIB)
        with bk.Context(window_bytes=4 * MIB, **kw) as ctx:
            ctx.register(buf, off)
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 18)) == oracle.wc(buf, off)
            st = ctx.stats()
        assert st["addr_elem_bytes"] == 1 and st["n_addresses"] == len(buf) and st["bytes_accessed"] == len(buf)
        if patterns:   # contiguous lanes: every lane is one stride-1 pattern
            assert st["n_pattern_lanes"] == st["n_addr_lanes"] and st["n_explicit_addr"] == 0
            assert st["bytes_addr"] < len(buf)
        else:
            assert st["bytes_addr"] >= 8 * len(buf)
        # grep (32-B keys in variable records: no pattern across records)
        gb, goff = gen.grep_records(n=30_000)
        with bk.Context(window_bytes=4 * MIB, **kw) as ctx:
            ctx.register(gb, goff)
            assert np.array_equal(ctx.grep(b"bigk", cap=len(goff)), oracle.grep(gb, goff, b"bigk"))
            assert ctx.stats()["addr_elem_bytes"] == 8
        # group-by sparse, k-means, k-mers, partition (fixed records)
        n = 60_000
        g = gen.groupby(n=n, stride=64)
        with bk.Context(window_bytes=4 * MIB, record_size=64, **kw) as ctx:
            ctx.register(g, None, n_records=n)
            c, q, a = ctx.groupby(4096)
            st = ctx.stats()
        wc_, wq, wa = oracle.groupby(g, n, 64, 4096)
        assert np.array_equal(c, wc_) and np.array_equal(q, wq) and np.allclose(a, wa, rtol=1e-5, atol=0)
        if patterns:   # 16 of 64 B per record, 8-B elements: strides (8, 56) recognised
            assert st["n_pattern_lanes"] == st["n_addr_lanes"]
        x = gen.points(n=n)
        with bk.Context(window_bytes=4 * MIB, record_size=64, **kw) as ctx:
            ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
            kc, ks, kchk = ctx.kmeans(x[:64])
        oc, os_, ochk, _ = oracle.kmeans(x, x[:64])
        assert np.array_equal(kc, oc) and kchk == ochk and np.allclose(ks, os_, rtol=1e-5, atol=0)
        d = gen.dna(n=8000)
        with bk.Context(window_bytes=4 * MIB, record_size=256, **kw) as ctx:
            ctx.register(d, None, n_records=8000)
            km, ct, _ = ctx.kmer(k=31, cap=1 << 20)
        okm, oct_ = oracle.kmer(d, 8000, k=31)
        o = np.argsort(km)
        assert np.array_equal(km[o], okm) and np.array_equal(ct[o], oct_)
        kv = gen.kv(n=n)
        with bk.Context(window_bytes=4 * MIB, record_size=16, **kw) as ctx:
            ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
            out, cc, bc = ctx.partition(1024)
        assert np.array_equal(bk.partition_materialize(out, cc), oracle.partition(kv, 1024)[1])


def test_addr_elem_bytes_config_and_errors():
    n = 20_000
    g = gen.groupby(n=n, stride=64)
    want = oracle.groupby(g, n, 64, 4096)
    for el in (1, 2, 4, 8, 16):
        with bk.Context(window_bytes=4 * MIB, record_size=64, gather_mode="addr", addr_elem_bytes=el) as ctx:
            ctx.register(g, None, n_records=n)
            c, q, a = ctx.groupby(4096)
            st = ctx.stats()
        assert np.array_equal(c, want[0]) and st["addr_elem_bytes"] == el and st["n_addresses"] == n * 16 // el
    with bk.Context(window_bytes=4 * MIB, record_size=64, gather_mode="addr", addr_elem_bytes=3) as ctx:
        ctx.register(g, None, n_records=n)
        with pytest.raises(bk.BkError) as e:
            ctx.groupby(4096)
        assert e.value.status == bk.BK_E_INVAL


class UserGen(C.Structure):
    _fields_ = [("rec_size", C.c_uint32), ("ext_off", C.c_uint32), ("ext_len", C.c_uint32), ("step", C.c_uint32),
                ("mode", C.c_int32), ("_pad", C.c_uint32), ("bad_addr", C.c_uint64)]


class UserUse(C.Structure):
    _fields_ = [("acc", C.c_void_p), ("ext_len", C.c_uint32), ("step", C.c_uint32), ("elem", C.c_uint32),
                ("variable", C.c_uint32)]


def _ulib():
    return C.CDLL(os.path.join(ROOT, "tests", "user", "libbkuser.so"))


def _mix64(x: int) -> int:
    x ^= x >> 30
    x = (x * 0xBF58476D1CE4E5B9) & M64
    x ^= x >> 27
    x = (x * 0x94D049BB133111EB) & M64
    return x ^ (x >> 31)


@pytest.mark.parametrize("step,patterns", [(1, True), (2, True), (1, False)])
def test_user_address_generator_fixed_records(step, patterns):
    """The generator walks each lane's records backwards and takes every `step`-th 4-B element of
    the 32-B field at +8: stages 2-3 must deliver exactly those elements in exactly that order."""
    n, R, eo, el, elem = 20_000, 64, 8, 32, 4
    data = gen.groupby(n=n, stride=R)
    lib = _ulib()
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    g = UserGen(R, eo, el, step, 0, 0, 0)
    u = UserUse(acc.data_ptr(), el, step, elem, 0)
    with bk.Context(window_bytes=2 * MIB, record_size=R, addr_elem_bytes=elem, no_patterns=not patterns) as ctx:
        ctx.register(data, None, n_records=n)
        ctx.run_user_addr(lib.user_gen, lib.user_use, gen_user=g, user=u, bound=[(eo, el)])
        st = ctx.stats()
    torch.cuda.synchronize()
    m = (el // elem + step - 1) // step
    want = 0
    v = data.view(np.uint32).reshape(n, R // 4)
    for e in range(m):
        col = (eo + e * step * elem) // 4
        vals = v[:, col].astype(np.uint64)
        for r in range(n):
            want = (want + _mix64((r << 8) ^ (e * step)) * (int(vals[r]) + 1)) & M64
    assert int(acc.item()) & M64 == want
    assert st["n_addresses"] == n * m and st["gather_mode"] == bk.BK_GATHER_ADDR
    if not patterns:
        assert st["n_explicit_addr"] == st["n_addresses"]


def test_user_address_generator_variable_records():
    gb, goff = gen.grep_records(n=20_000)
    lib = _ulib()
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    g = UserGen(0, 0, 0, 1, 0, 0, 0)
    u = UserUse(acc.data_ptr(), 0, 1, 8, 1)
    with bk.Context(window_bytes=2 * MIB, addr_elem_bytes=8) as ctx:
        ctx.register(gb, goff)
        ctx.run_user_addr(lib.user_gen, lib.user_use, gen_user=g, user=u, bound=[(8, 8), (16, 8)])
    torch.cuda.synchronize()
    raw = gb.tobytes()
    want = 0
    for r, s in enumerate(goff.astype(np.int64)):
        key = int.from_bytes(raw[s + 16: s + 24], "little")
        rid = int.from_bytes(raw[s + 8: s + 16], "little")
        want = (want + _mix64(r) * ((key ^ rid) + 1)) & M64
    assert int(acc.item()) & M64 == want


@pytest.mark.parametrize("mode", [1, 2])
def test_user_address_generator_errors(mode):
    n = 5000
    data = gen.groupby(n=n, stride=64)
    lib = _ulib()
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    g = UserGen(64, 0, 16, 1, mode, 0, n * 64)   # mode 1: address == nbytes (outside); 2: count > capacity
    u = UserUse(acc.data_ptr(), 16, 1, 8, 0)
    with bk.Context(window_bytes=1 * MIB, record_size=64) as ctx:
        ctx.register(data, None, n_records=n)
        with pytest.raises(bk.BkError) as e:
            ctx.run_user_addr(lib.user_gen, lib.user_use, gen_user=g, user=u, bound=[(0, 16)])
        assert e.value.status == bk.BK_E_INVAL
        c, q, a = ctx.groupby(4096)   # the context stays usable
    assert int(c.sum()) == n
