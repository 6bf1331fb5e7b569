"""CPU test of the product's host-side assembly (csrc/host_gather.cpp, BK_GATHER_CPU/HYBRID):
compiled into a small harness with g++ (no GPU needed) and compared byte for byte with the
oracle's layout definition (O-L) on grep keys, sparse fixed records, whole records and
multi-extent specs."""
import os
import subprocess
import textwrap

import numpy as np
import pytest

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_ipps_mokhtaris14_b200", "csrc")
HARNESS = textwrap.dedent(r'''
    #include "host_gather.h"
    #include <cstdio>
    #include <cstdlib>
    #include <vector>
    // argv: data.bin off.bin(or -) n rec_size lo hi L n_ext [off len]... out.bin threads
    int main(int argc, char** argv) {
      using namespace bk;
      auto slurp = [](const char* p, std::vector<uint8_t>& v) {
        FILE* f = fopen(p, "rb"); fseek(f, 0, SEEK_END); long n = ftell(f); fseek(f, 0, SEEK_SET);
        v.resize(n); if (n) fread(v.data(), 1, n, f); fclose(f); };
      std::vector<uint8_t> data, offb;
      slurp(argv[1], data);
      const bool has_off = argv[2][0] != '-';
      if (has_off) slurp(argv[2], offb);
      const uint64_t n = strtoull(argv[3], 0, 10), rs = strtoull(argv[4], 0, 10);
      const uint64_t lo = strtoull(argv[5], 0, 10), hi = strtoull(argv[6], 0, 10);
      const uint32_t L = strtoul(argv[7], 0, 10), ne = strtoul(argv[8], 0, 10);
      Access a{}; a.whole = ne == 0; a.n_ext = ne;
      for (uint32_t e = 0; e < ne; ++e) { a.ext_off[e] = strtoul(argv[9 + 2 * e], 0, 10);
        a.ext_len[e] = strtoul(argv[10 + 2 * e], 0, 10); a.E += a.ext_len[e]; }
      const char* out = argv[9 + 2 * ne];
      const int threads = atoi(argv[10 + 2 * ne]);
      const uint64_t* off = has_off ? (const uint64_t*)offb.data() : nullptr;
      HostData d{data.data(), off, n, data.size(), rs};
      auto start = [&](uint64_t r) { return off ? (r < n ? off[r] : data.size()) : r * rs; };
      Chunk c{}; c.lo = lo; c.hi = hi; c.base_byte = start(lo); c.end_byte = start(hi); c.L = L; c.ntiles = L / 32;
      c.accessed = a.whole ? c.end_byte - c.base_byte : (hi - lo) * a.E;
      HostPool pool(threads);
      std::vector<uint8_t> st(64 << 20);
      std::vector<uint64_t> f, t;
      const uint64_t sz = host_gather_chunk(pool, d, a, c, st.data(), st.size(), f, t);
      FILE* fo = fopen(out, "wb"); fwrite(st.data(), 1, sz, fo); fclose(fo);
      return 0;
    }
''')


@pytest.fixture(scope="module")
def harness(tmp_path_factory):
    d = tmp_path_factory.mktemp("hg")
    src = d / "h.cpp"
    src.write_text(HARNESS)
    exe = d / "h"
    cuda_inc = "/usr/local/cuda/include"
    subprocess.check_call(["g++", "-std=c++17", "-O2", "-march=x86-64-v3", f"-I{cuda_inc}", f"-I{CSRC}", str(src),
                           os.path.join(CSRC, "host_gather.cpp"), "-o", str(exe), "-lpthread"])
    return exe, d


CASES = [
    ("grep", [(16, 32)], 0, 96),
    ("grep_multi", [(16, 8), (40, 8)], 0, 64),
    ("text_whole", None, 0, 160),
    ("sparse64", [(0, 16)], 64, 128),
    ("points_whole", None, 64, 32),
    ("dup", [(8, 4), (0, 12), (8, 4)], 16, 64),
]


@pytest.mark.parametrize("name,extents,rs,L", CASES)
@pytest.mark.parametrize("threads", [1, 5])
def test_host_gather_matches_layout_oracle(harness, name, extents, rs, L, threads):
    exe, d = harness
    if name.startswith("grep"):
        buf, off = gen.grep_records(n=3000)
    elif name == "text_whole":
        buf, off = gen.text(cap_bytes=40000)
    elif name == "points_whole":
        buf, off = gen.points(n=1500).view(np.uint8).reshape(-1), None
    else:
        buf, off = gen.groupby(n=2000, stride=rs), None
    n = len(off) if off is not None else len(buf) // rs
    (d / "data.bin").write_bytes(buf.tobytes())
    if off is not None:
        (d / "off.bin").write_bytes(off.tobytes())
    for lo, hi in [(0, n // 3), (n // 3 + 1, n), (5, 5)]:
        args = [str(exe), str(d / "data.bin"), str(d / "off.bin") if off is not None else "-", str(n), str(rs),
                str(lo), str(hi), str(L), str(len(extents or []))]
        for eo, el in extents or []:
            args += [str(eo), str(el)]
        args += [str(d / "out.bin"), str(threads)]
        subprocess.check_call(args)
        stage, _, _, _ = oracle.layout(buf, off, n, len(buf), rs, extents, lo, hi, L)
        assert (d / "out.bin").read_bytes() == stage.tobytes(), (name, lo, hi)


PACK_HARNESS = textwrap.dedent(r'''
    #include "host_gather.h"
    #include <cstdio>
    #include <cstdlib>
    #include <vector>
    // argv: data.bin off.bin(or -) n rec_size lo hi ext_off ext_len dst_shift out.bin threads
    int main(int argc, char** argv) {
      using namespace bk;
      auto slurp = [](const char* p, std::vector<uint8_t>& v) {
        FILE* f = fopen(p, "rb"); fseek(f, 0, SEEK_END); long n = ftell(f); fseek(f, 0, SEEK_SET);
        v.resize(n); if (n) fread(v.data(), 1, n, f); fclose(f); };
      std::vector<uint8_t> data, offb;
      slurp(argv[1], data);
      const bool has_off = argv[2][0] != '-';
      if (has_off) slurp(argv[2], offb);
      const uint64_t n = strtoull(argv[3], 0, 10), rs = strtoull(argv[4], 0, 10);
      const uint64_t lo = strtoull(argv[5], 0, 10), hi = strtoull(argv[6], 0, 10);
      Access a{}; a.n_ext = 1; a.ext_off[0] = strtoul(argv[7], 0, 10); a.ext_len[0] = strtoul(argv[8], 0, 10);
      a.E = a.ext_len[0];
      const uint64_t shift = strtoull(argv[9], 0, 10);
      HostData d{data.data(), has_off ? (const uint64_t*)offb.data() : nullptr, n, data.size(), rs};
      Chunk c{}; c.lo = lo; c.hi = hi;
      HostPool pool(atoi(argv[11]));
      uint8_t* st = (uint8_t*)aligned_alloc(64, 64 << 20);
      const uint64_t sz = host_pack_chunk(pool, d, a, c, st + shift, (64 << 20) - shift, 1000);
      FILE* fo = fopen(argv[10], "wb"); fwrite(st + shift, 1, sz, fo); fclose(fo);
      return 0;
    }
''')


@pytest.fixture(scope="module")
def pack_harness(tmp_path_factory):
    d = tmp_path_factory.mktemp("hp")
    src = d / "p.cpp"
    src.write_text(PACK_HARNESS)
    exe = d / "p"
    subprocess.check_call(["g++", "-std=c++17", "-O2", "-march=x86-64-v3", "-I/usr/local/cuda/include", f"-I{CSRC}",
                           str(src), os.path.join(CSRC, "host_gather.cpp"), "-o", str(exe), "-lpthread"])
    return exe, d


@pytest.mark.parametrize("cfg", ["1", "2", "3", "4", "5", "6", "7", "8"])
@pytest.mark.parametrize("field", ["grep_key", "sparse16", "dna96"])
def test_host_pack_chunk_every_config(pack_harness, cfg, field):
    """The HYBRID / CPU-mode packer (host_pack_chunk, every BK_PACK_CFG: prefetch distances; 7, 8 with
    32-B AVX2 copies) writes each record's accessed field, in record order, and nothing else — for a
    32-B aligned destination and a 16-B aligned one (where the 32-B configurations fall back)."""
    exe, d = pack_harness
    if field == "grep_key":
        buf, off = gen.grep_records(n=5000)
        rs, eo, el = 0, 16, 32
    elif field == "sparse16":
        buf, off = gen.groupby(n=7000, stride=64), None
        rs, eo, el = 64, 0, 16
    else:
        buf, off = gen.dna(n=3000), None
        rs, eo, el = 256, 16, 96
    n = len(off) if off is not None else len(buf) // rs
    (d / "data.bin").write_bytes(buf.tobytes())
    if off is not None:
        (d / "off.bin").write_bytes(off.tobytes())
    starts = off.astype(np.int64) if off is not None else np.arange(n, dtype=np.int64) * rs
    env = dict(os.environ, BK_PACK_CFG=cfg)
    for lo, hi in [(0, n), (7, n - 3), (4, 4)]:
        for shift in (0, 16):
            subprocess.check_call([str(exe), str(d / "data.bin"), str(d / "off.bin") if off is not None else "-",
                                   str(n), str(rs), str(lo), str(hi), str(eo), str(el), str(shift),
                                   str(d / "out.bin"), "3"], env=env)
            want = b"".join(buf[s + eo: s + eo + el].tobytes() for s in starts[lo:hi])
            assert (d / "out.bin").read_bytes() == want, (field, cfg, lo, hi, shift)
