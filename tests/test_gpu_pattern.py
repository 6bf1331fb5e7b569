"""GPU parity of the online pattern recognition of stage 1 (NEXT f2) against
the oracle's online rule, lane by lane, on the address streams of four access specs."""
import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu
MIB = 1 << 20


def lane_addresses(buf_len, off, rs, extents, first, nrec, n, elem):
    addrs = []
    for r in range(first, first + nrec):
        s = int(off[r]) if off is not None else r * rs
        e = (int(off[r + 1]) if r + 1 < n else buf_len) if off is not None else s + rs
        for eo, el in (extents or [(0, e - s)]):
            addrs.extend(range(s + eo, s + eo + el, elem))
    return addrs


CASES = [
    ("wc_bytes", None, 1, 8),
    ("kmeans_fp32", None, 4, 8),
    ("groupby_sparse_fields", [(0, 16)], 4, 8),
    ("grep_key_words", [(16, 32)], 4, 8),
    ("kmeans_short_buffer", None, 4, 2),
]


@pytest.mark.parametrize("name,extents,elem,T", CASES)
def test_pattern_lanes_match_oracle(name, extents, elem, T):
    if name.startswith("wc"):
        buf, off = gen.text(cap_bytes=200_000)
        rs = 0
    elif name.startswith("kmeans"):
        buf, off, rs = gen.points(n=20_000).view(np.uint8).reshape(-1), None, 64
    elif name.startswith("groupby"):
        buf, off, rs = gen.groupby(n=30_000, stride=64), None, 64
    else:
        buf, off = gen.grep_records(n=20_000)
        rs = 0
    n = len(off) if off is not None else len(buf) // rs
    with bk.Context(window_bytes=4 * MIB, gather_mode="zc", chunk_bytes=65536, lanes=64, record_size=rs) as ctx:
        ctx.register(buf, off, n_records=n)
        plan = oracle.plan_chunks(off, n, len(buf), rs, extents, 65536)
        c = len(plan) // 2 - 1
        tot, (lp, lst, lbase, lcnt) = ctx.pattern_stats(extents, elem_bytes=elem, T=T, chunk=c)
    _, lf, ln, _ = oracle.layout(buf, off, n, len(buf), rs, extents, int(plan[c]), int(plan[c + 1]), 64,
                                 with_stage=False)
    pattern_lanes = 0
    for t in range(64):
        a = lane_addresses(len(buf), off, rs, extents, int(lf[t]), int(ln[t]), n, elem)
        want = oracle.pattern_online(a, T=T, pmax=4)
        assert int(lcnt[t]) == len(a)
        if want is None:
            assert lp[t] == 0, (t, lp[t], lst[t])
        else:
            pattern_lanes += 1
            assert lp[t] == len(want[1]) and int(lbase[t]) == want[0], t
            assert list(lst[t][: lp[t]]) == want[1]
    # every accessed element of every record is one address, over all chunks
    per_rec = [(int(off[r + 1]) if r + 1 < n else len(buf)) - int(off[r]) for r in range(n)] if extents is None and off is not None \
        else [rs if extents is None else sum(x[1] for x in extents)] * n
    assert tot["n_addresses"] == sum(-(-b // elem) for b in per_rec)
    if name in ("wc_bytes", "kmeans_fp32", "groupby_sparse_fields"):
        assert pattern_lanes >= 60  # contiguous / fixed-stride streams reduce to patterns
        assert tot["pattern_bytes"] < tot["address_bytes"] / 10
    if name == "grep_key_words":
        assert pattern_lanes == 0    # variable-length records: no periodic key addresses
    if name == "kmeans_short_buffer":
        assert pattern_lanes == 0    # T = 2 leaves no delta to confirm a period: all explicit
        assert tot["pattern_bytes"] == tot["address_bytes"]
