"""bk_run_user: the caller's own stage-4 kernel over the staged chunks (include/bk.h), written only
against the public layout (tests/user/user_kernels.cu). The checksum it accumulates must equal the
one computed here from the host data set, in every gather mode, for field extents and for whole
variable-length records; a failing callback aborts the run with BK_E_INVAL."""
import ctypes as C
import os

import numpy as np
import pytest
import torch

import gen
from paper_conf_ipps_mokhtaris14_b200 import bk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MIB = 1 << 20
M64 = (1 << 64) - 1


class UserSum(C.Structure):
    _fields_ = [("acc", C.c_void_p), ("E", C.c_uint32), ("fail_at", C.c_int32), ("calls", C.c_uint64)]


def _ulib():
    so = os.path.join(ROOT, "tests", "user", "libbkuser.so")
    assert os.path.exists(so), "tests/user/libbkuser.so not built (make)"
    return C.CDLL(so)


def _mix64_np(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64)
    with np.errstate(over="ignore"):
        x ^= x >> np.uint64(30)
        x *= np.uint64(0xBF58476D1CE4E5B9)
        x ^= x >> np.uint64(27)
        x *= np.uint64(0x94D049BB133111EB)
        x ^= x >> np.uint64(31)
    return x


def expected(buf: np.ndarray, off, n: int, rec_size: int, extents) -> int:
    """sum_r mix64(r) * (1 + sum of r's accessed bytes), mod 2^64 (duplicated extents count twice)."""
    starts = np.arange(n, dtype=np.uint64) * np.uint64(rec_size) if off is None else off.astype(np.uint64)
    b = buf.astype(np.uint64)
    if extents:
        s = np.zeros(n, np.uint64)
        for eo, el in extents:
            for x in range(el):
                s += b[(starts + np.uint64(eo + x)).astype(np.int64)]
    else:
        ends = np.append(starts[1:], np.uint64(len(buf)))
        cs = np.concatenate([np.zeros(1, np.uint64), np.cumsum(b, dtype=np.uint64)])
        s = cs[ends.astype(np.int64)] - cs[starts.astype(np.int64)]
    with np.errstate(over="ignore"):
        tot = (_mix64_np(np.arange(n, dtype=np.uint64)) * (s + np.uint64(1))).sum(dtype=np.uint64)
    return int(tot)


def _run(ctx, extents, E, fail_at=-1, lane_bytes=0):
    acc = torch.zeros(1, dtype=torch.int64, device="cuda")
    u = UserSum(acc.data_ptr(), E, fail_at, 0)
    ctx.run_user(_ulib().user_sum_chunk, u, extents=extents, lane_bytes=lane_bytes)
    return int(acc.item()) & M64, u.calls


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["zc", "dense", "cpu", "hybrid"])
def test_user_kernel_field_extents(mode):
    n = 200_003
    buf = gen.groupby(n=n, stride=64)
    for extents in ([(0, 16)], [(8, 8), (0, 4), (8, 8)]):
        E = sum(l for _, l in extents)
        want = expected(buf, None, n, 64, extents)
        with bk.Context(window_bytes=2 * MIB, gather_mode=mode, record_size=64) as ctx:
            ctx.register(buf, None, n_records=n)
            got, calls = _run(ctx, extents, E)
            st = ctx.stats()
        assert got == want, (mode, extents)
        assert calls == st["n_chunks"] >= 4
        assert st["bytes_accessed"] == E * n


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["zc", "dense", "cpu"])
def test_user_kernel_whole_variable_records(mode):
    buf, off = gen.text(cap_bytes=3 * MIB)
    want = expected(buf, off, len(off), 0, None)
    with bk.Context(window_bytes=512 * 1024, n_slots=3, gather_mode=mode) as ctx:
        ctx.register(buf, off)
        got, calls = _run(ctx, None, 0, lane_bytes=512)
        got2, _ = _run(ctx, None, 0)    # runs again (never graph-replayed: the callback runs each time)
    assert got == want == got2 and calls >= 4


@pytest.mark.gpu
def test_user_kernel_callback_failure_and_errors():
    n = 100_000
    buf = gen.groupby(n=n, stride=16)
    with bk.Context(window_bytes=1 * MIB, record_size=16) as ctx:
        ctx.register(buf, None, n_records=n)
        with pytest.raises(bk.BkError) as e:
            _run(ctx, [(0, 16)], 16, fail_at=2)
        assert e.value.status == bk.BK_E_INVAL
        with pytest.raises(bk.BkError) as e:
            _run(ctx, [(8, 16)], 16)          # extent past the 16-B record
        assert e.value.status == bk.BK_E_INVAL
        got, _ = _run(ctx, [(0, 16)], 16)     # the context stays usable
        assert got == expected(buf, None, n, 16, [(0, 16)])
