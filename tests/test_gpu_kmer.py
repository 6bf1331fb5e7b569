"""GPU parity of f4 (k-mer counting over DNA read records) against oracle O6."""
import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu
MIB = 1 << 20


def sorted_pairs(km, ct):
    o = np.argsort(km)
    return km[o], ct[o]


@pytest.mark.parametrize("k,mode", [(31, "hybrid"), (21, "zc"), (13, "dense"), (31, "cpu"), (1, "zc")])
def test_kmer_matches_oracle(k, mode):
    n = 40_000
    buf = gen.dna(n=n, genome_len=1 << 18, err_pm=2, n_pm=3)
    wk, wc = oracle.kmer(buf, n, k)
    with bk.Context(window_bytes=2 * MIB, gather_mode=mode, record_size=256) as ctx:
        ctx.register(buf, None, n_records=n)
        km, ct, total = ctx.kmer(k=k, table_slots=1 << 22)
        st = ctx.stats()
    assert st["n_chunks"] >= 4
    gk, gc = sorted_pairs(km, ct)
    assert np.array_equal(gk, wk) and np.array_equal(gc, wc)
    assert total == int(wc.sum())
    if mode == "zc":
        assert st["bytes_accessed"] == 96 * n   # 37.5% of the 256-B records (Table I DNA: 36%)


def test_kmer_errors():
    buf = gen.dna(n=1000)
    with bk.Context(window_bytes=1 * MIB, record_size=256) as ctx:
        ctx.register(buf, None, n_records=1000)
        for kw in ({"k": 0}, {"k": 32}, {"seq_len": 90}, {"seq_off": 200}, {"table_slots": 1000}):
            with pytest.raises(bk.BkError):
                ctx.kmer(**kw)
        with pytest.raises(bk.BkError) as e:
            ctx.kmer(k=31, table_slots=1 << 10)
        assert e.value.status == bk.BK_E_CAPACITY
