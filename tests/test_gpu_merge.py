"""bk_merge_counts (the GPU merge of all-gathered per-rank count tables) against a
plain dict merge: per key the counts sum, every other word comes from the key's first row in
(segment, row) order; padded segments are ignored past seg_rows; capacity errors report the size."""
import numpy as np
import pytest

from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu


def ref_merge(rows, seg_rows, stride, key_u64, count_col):
    out = {}
    for s, n in enumerate(seg_rows):
        for r in rows[s * stride: s * stride + n]:
            k = tuple(int(x) for x in r[:key_u64])
            if k in out:
                out[k][count_col] = (out[k][count_col] + int(r[count_col])) % (1 << 64)
            else:
                out[k] = [int(x) for x in r]
    return sorted(tuple(v) for v in out.values())


@pytest.mark.parametrize("W,key_u64,count_col", [(6, 3, 3), (2, 1, 1), (5, 2, 4)])
@pytest.mark.parametrize("segs", [[0], [1], [1000, 0, 17], [4096, 4096, 4000, 1, 333, 4096, 2048, 5]])
def test_merge_counts_matches_dict(W, key_u64, count_col, segs):
    import torch
    rng = np.random.default_rng(len(segs) * 100 + W)
    stride = max(max(segs), 1)
    nkeys = max(sum(segs) // 3, 1)
    keys = rng.integers(0, 1 << 63, size=(nkeys, key_u64), dtype=np.int64)
    keys[0] = 0                                   # an all-zero key is a key like any other
    rows = rng.integers(0, 1 << 40, size=(len(segs) * stride, W), dtype=np.int64)
    pick = rng.integers(0, nkeys, size=len(rows))
    rows[:, :key_u64] = keys[pick]
    ref = ref_merge(rows.astype(np.uint64), segs, stride, key_u64, count_col)
    with bk.Context(window_bytes=1 << 20) as ctx:
        g = torch.from_numpy(rows).cuda()
        out = torch.full((max(len(ref), 1), W), -1, dtype=torch.int64, device="cuda")
        m = ctx.merge_counts(g, segs, stride, W, key_u64, count_col, out)
        assert m == len(ref)
        got = sorted(tuple(int(x) for x in r) for r in out[:m].cpu().numpy().astype(np.uint64))
        assert got == ref
        if len(ref) > 1:   # one short: BK_E_CAPACITY with the needed size
            small = torch.empty((len(ref) - 1, W), dtype=torch.int64, device="cuda")
            with pytest.raises(bk.BkError) as e:
                ctx.merge_counts(g, segs, stride, W, key_u64, count_col, small)
            assert e.value.status == bk.BK_E_CAPACITY


def test_merge_counts_rejects_bad_layouts():
    import torch
    g = torch.zeros(8, 4, dtype=torch.int64, device="cuda")
    out = torch.zeros(8, 4, dtype=torch.int64, device="cuda")
    with bk.Context(window_bytes=1 << 20) as ctx:
        for args in ([4], 2, 4, 0, 1), ([4], 2, 4, 2, 1), ([4], 2, 4, 2, 4), ([3], 2, 4, 1, 2):
            segs, stride, W, k, cc = args
            with pytest.raises(bk.BkError) as e:
                ctx.merge_counts(g, segs, stride, W, k, cc, out)
            assert e.value.status == bk.BK_E_INVAL
