"""Pins for oracle O1 (word count)."""
from collections import Counter

import numpy as np
import pytest

import gen
import oracle
from _pins import words_of_record


def records(*recs: bytes):
    buf = b"".join(recs)
    off = np.cumsum([0] + [len(r) for r in recs[:-1]]).astype(np.uint64) if recs else np.zeros(0, np.uint64)
    return buf, off


def brute(buf: bytes, off) -> list:
    """Independent formulation: bytes.split per record + Counter, sorted by bytes order."""
    off = [int(o) for o in off]
    c = Counter()
    for i, s in enumerate(off):
        e = off[i + 1] if i + 1 < len(off) else len(buf)
        c.update(words_of_record(buf[s:e]))
    return sorted(c.items())


def test_bytes_split_is_the_c_locale_isspace_set():
    # the pin helper's delimiter set must be exactly {0x20, 0x09-0x0D}
    for b in range(256):
        assert (len(bytes([65, b, 66]).split()) == 2) == (b in b" \t\n\x0b\x0c\r"), b


def test_adversarial_catalogue():
    cases = [
        (b"a b  c\t\r\n",),
        (b"  \t\r\n",),
        (b"", b"", b"x"),
        (b"\x00\x80\xff word\n", b"\x00\x80\xff"),
        (b"last line without newline",),
        (b"ab", b"cd"),  # record boundary is a delimiter (A19): two words, not "abcd"
        (b"dup dup dup\n", b"dup\n"),
        (b"z a aa a ab b\n",),
    ]
    for recs in cases:
        buf, off = records(*recs)
        assert oracle.wc(buf, off) == brute(buf, off), recs


def test_record_boundary_splits_words():
    buf, off = records(b"ab", b"cd")
    assert oracle.wc(buf, off) == [(b"ab", 1), (b"cd", 1)]


def test_memcmp_order_shorter_prefix_first():
    buf, off = records(b"ab a abc b \x80 A\n")
    assert [w for w, _ in oracle.wc(buf, off)] == [b"A", b"a", b"ab", b"abc", b"b", b"\x80"]


def test_repeated_word_and_all_delimiters_and_empty():
    buf, off = records(b"w " * 37 + b"\n")
    assert oracle.wc(buf, off) == [(b"w", 37)]
    buf, off = records(b" \t\n\r\x0b\x0c", b"\n")
    assert oracle.wc(buf, off) == []
    assert oracle.wc(b"", np.zeros(0, np.uint64)) == []


def test_generated_text_vs_brute_force_and_rescan():
    buf, off = gen.text(cap_bytes=20000)
    b = buf.tobytes()
    got = oracle.wc(buf, off)
    assert got == brute(b, off)
    # O(n*V) rescan for every distinct word: count occurrences as whole words per record
    recs = [b[int(off[i]): int(off[i + 1]) if i + 1 < len(off) else len(b)] for i in range(len(off))]
    for w, c in got[:50]:
        assert c == sum(r.split().count(w) for r in recs)


def test_total_equals_delimiter_transitions():
    buf, off = gen.text(cap_bytes=200000)
    b = buf.tobytes()
    total = sum(c for _, c in oracle.wc(buf, off))
    # a word starts at every non-delimiter byte whose predecessor is a delimiter or a record start
    starts = set(int(o) for o in off)
    delim = set(b" \t\n\x0b\x0c\r")
    n = sum(1 for i, ch in enumerate(b) if ch not in delim and (i in starts or b[i - 1] in delim))
    assert total == n


@pytest.mark.parametrize("cap", [1 << 12, 1 << 16])
def test_generator_shape(cap):
    buf, off = gen.text(cap_bytes=cap)
    assert len(buf) <= cap and off[0] == 0 and np.all(np.diff(off.astype(np.int64)) > 0)
    assert buf[-1] == ord("\n")
