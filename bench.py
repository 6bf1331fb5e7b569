#!/usr/bin/env python3
"""bench.py — BigKernel out-of-core streaming throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload grep|wordcount|groupby|kmeans] [--gather auto|zc|dense]

Default workload = BASELINE.json configs[1]: grep/filter over 16 GiB of seeded variable-length
records through a 2 GiB device window (the config the metric is quoted on that fits one GPU;
configs[0], 64 MiB word count, is the small oracle case). One "step" = one bk_run over the
whole data set: every §8(a) row (chunk plan, address generation, zero-copy gather, compute,
ordered compaction, finalize + D2H) plus, for N>1, the NCCL exchange of match counts.

Data live in pinned host memory (registered once, outside the timed region): the method
streams them over PCIe every step, so there is no "HBM-resident input" variant; 16 GiB per
GPU is > 126 MB L2, so no L2 flush is needed between steps. Under torchrun each rank streams
its own contiguous record range (weak scaling, 16 GiB per GPU).

--impl reference times the CPU oracle (oracle/, single-threaded C) on the host cores over a
bounded sample per step; rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402

GIB = 1 << 30
MIB = 1 << 20
HUGE = True  # data sets in 2 MiB-aligned mappings with transparent huge pages (--pages)
METRIC = "input GB/s streamed out-of-core at 1/2/4/8 B200; % of host-link roofline"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference", "dbuf", "sbuf"],
                    help="ours | reference (CPU oracle) | dbuf / sbuf (the paper's GPU double / single "
                         "buffering variants, for ablations)")
    ap.add_argument("--workload", default="grep", choices=["grep", "wordcount", "groupby", "groupby_sparse", "kmeans",
                                                             "partition", "kmer"])
    ap.add_argument("--gather", default="auto", choices=["auto", "zc", "dense", "cpu", "hybrid", "fused", "addr"])
    ap.add_argument("--gib", type=float, default=None, help="per-GPU data size override (GiB)")
    ap.add_argument("--window-mib", type=int, default=None)
    ap.add_argument("--slots", type=int, default=0)
    ap.add_argument("--host-threads", type=int, default=0)
    ap.add_argument("--lane-bytes", type=int, default=0)
    ap.add_argument("--zc-share", type=int, default=0, help="HYBRID zero-copy share of chunks, per mille")
    ap.add_argument("--K", type=int, default=64, help="k-means clusters (C3: 64)")
    ap.add_argument("--pages", default="numpy", choices=["huge", "4k", "numpy"],
                    help="host data set pages: THP-backed mapping, 4 KiB mapping, or plain numpy")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-dbuf", action="store_true", help="skip the double-buffering baseline measurement")
    ap.add_argument("--no-profile", action="store_true", help="disable per-stage event timing")
    ap.add_argument("--no-trace", action="store_true", help="skip the CUPTI-traced pass (BK_FLAG_TRACE)")
    ap.add_argument("--dump", default=None, help="after the timed steps, run one more step and write this rank's "
                                                 "(merged) result to DUMP/rank<r>.npz (the N>1 parity tests)")
    args = ap.parse_args()
    if args.slots == 0 and args.workload == "wordcount":
        args.slots = 8   # the 8 MiB window: more, smaller chunks in flight (profiles/r01_wc_sweep.md)
    if args.slots == 0 and args.workload == "partition":
        args.slots = 12  # smaller chunks shorten the one-direction fill and drain (profiles/r02_partition.md)
    return args


# ------------------------------------------------------------------------------ workloads
WORKLOADS = {
    # name: (default GiB per GPU, window MiB, config string)
    "grep": (16.0, 2048, "C2 grep/filter: variable-length records (48-464 B, mean 256), 32-B key at +16, "
                         "pattern 'bigk' (1% planted), ordered match indices"),
    "wordcount": (64 / 1024, 8, "C1 word count: Zipf(1.0) text lines, 65,536-word vocabulary"),
    "groupby": (16.0, 2048, "C5 group-by sum: {u32 key<4096, u32 qty, f64 amount} 16-B records"),
    "groupby_sparse": (16.0, 2048, "C5 sparse variant: the same 16 B inside 64-B records (25% read, like Table I "
                                   "MCA-indexed P:929)"),
    "kmeans": (16.0, 2048, "C3 k-means step: 16-dim fp32 points, K=64, Forgy init"),
    "kmer": (4.0, 2048, "f4 k-mer counting (k=31) over 256-B DNA read records, 96-base sequence at +16 (37.5% "
                        "read, Table I DNA: 36%), reads of a seeded 2^25-base genome, 0.1% substitutions, 0.2% N"),
    "partition": (8.0, 2048, "C4 stable hash partition: {u64 key, u64 value} 16-B records into 1024 buckets, "
                             "bucket-sorted chunks written back to host (full duplex)"),
}


def _cpulist(text: str) -> list[int]:
    out = []
    for part in text.strip().split(","):
        if "-" in part:
            a, b = part.split("-")
            out.extend(range(int(a), int(b) + 1))
        elif part:
            out.append(int(part))
    return out


def numa_local_cores(torch, local: int) -> list[int] | None:
    """Host cores for this rank when several ranks share the node: the cores PCIe-local to its GPU
    (sysfs local_cpulist), split evenly among the ranks whose GPUs share that list, so that first
    touch of the shard lands on the GPU's NUMA node and the assembly pools do not oversubscribe."""
    lists = []
    for d in range(torch.cuda.device_count()):
        p = torch.cuda.get_device_properties(d)
        path = f"/sys/bus/pci/devices/{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0/local_cpulist"
        try:
            with open(path) as f:
                cores = _cpulist(f.read())
        except OSError:
            return None
        lists.append(tuple(c for c in cores if c in os.sched_getaffinity(0)))
    mine = lists[local]
    peers = [d for d, l in enumerate(lists) if l == mine]
    k, m = peers.index(local), len(peers)
    part = list(mine[len(mine) * k // m: len(mine) * (k + 1) // m])
    return part or None


def make_shard(workload: str, gib: float, rank: int, world: int, K: int = 64):
    """Rank r's contiguous shard of the weak-scaled data set. Returns dict."""
    nbytes = int(gib * GIB)
    if workload == "grep":
        first = 0
        for r in range(rank):
            first += gen.grep_count_for_bytes(gen.SEED_GREP, first, nbytes)
        buf, off = gen.grep_records(gen.SEED_GREP, first=first, max_bytes=nbytes,
                                    out=gen.alloc(nbytes, huge=HUGE) if HUGE is not None else None)
        return dict(buf=buf, off=off, n=len(off), first=first, rec_size=0)
    if workload == "wordcount":
        buf, off = gen.text(gen.SEED_WC + rank, cap_bytes=nbytes)
        return dict(buf=buf, off=off, n=len(off), first=0, rec_size=0)
    if workload in ("groupby", "groupby_sparse"):
        stride = 16 if workload == "groupby" else 64
        n = nbytes // stride
        buf = gen.groupby(gen.SEED_GROUPBY, first=rank * n, n=n, stride=stride,
                          out=gen.alloc(n * stride, huge=HUGE) if HUGE is not None else None)
        return dict(buf=buf, off=None, n=n, first=rank * n, rec_size=stride)
    if workload == "kmer":
        n = nbytes // 256
        buf = gen.dna(gen.SEED_DNA, first=rank * n, n=n, genome_len=1 << 25, err_pm=1, n_pm=2)
        return dict(buf=buf, off=None, n=n, first=rank * n, rec_size=256)
    if workload == "partition":
        n = nbytes // 16
        kv = gen.kv(gen.SEED_KV, first=rank * n, n=n)
        return dict(buf=kv.view(np.uint8).reshape(-1), off=None, n=n, first=rank * n, rec_size=16,
                    out=np.empty((n, 2), np.uint64))
    n = nbytes // 64
    x = gen.points(gen.SEED_KMEANS, first=rank * n, n=n)
    return dict(buf=x.view(np.uint8).reshape(-1), off=None, n=n, first=rank * n, rec_size=64,
                mu=gen.points(gen.SEED_KMEANS, first=0, n=K))


# ------------------------------------------------------------------------------ helpers
class ClockSampler:
    """SM clocks + throttle reasons sampled every 10 ms through NVML while the timed region runs
    (the nvidia-smi query of the profiling recipe, without its ~100 ms start-up, so that short
    regions are sampled too); one sample is taken on entry and one on exit of the region."""

    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))

    def __init__(self, dev: int):
        self.dev, self.rows, self.h, self.stop = dev, [], None, threading.Event()

    def _sample(self):
        import pynvml
        sm = pynvml.nvmlDeviceGetClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        mx = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        rs = pynvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        self.rows.append((sm, mx, rs))

    def _loop(self):
        while not self.stop.wait(0.01):
            self._sample()

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
            ids = [x for x in vis.split(",") if x.strip()]
            idx = int(ids[self.dev]) if ids and ids[self.dev].strip().isdigit() else self.dev
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self._sample()
            self.t = threading.Thread(target=self._loop, daemon=True)
            self.t.start()
        except Exception:
            self.h = None
        return self

    def __exit__(self, *a):
        if self.h is not None:
            self.stop.set()
            self.t.join(timeout=5)
            try:
                self._sample()
            except Exception:
                pass

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        reasons = sorted({n for r in self.rows for n, bit in self.REASONS if r[2] & bit})
        return {"sm_mhz": statistics.median(r[0] for r in self.rows), "sm_max_mhz": max(r[1] for r in self.rows),
                "reasons": reasons, "samples": len(self.rows), "how": "NVML every 10 ms during the timed steps"}


def measure_h2d_peak(torch, dev) -> float:
    """Pinned H2D DMA bandwidth (GB/s), 1 GiB in 256 MiB copies, best of 3: the host-link roofline."""
    src = torch.empty(GIB, dtype=torch.uint8, pin_memory=True)
    dst = torch.empty(GIB, dtype=torch.uint8, device=dev)
    best = 0.0
    for _ in range(4):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for o in range(0, GIB, 256 * MIB):
            dst[o:o + 256 * MIB].copy_(src[o:o + 256 * MIB], non_blocking=True)
        b.record()
        b.synchronize()
        best = max(best, GIB / (a.elapsed_time(b) * 1e-3) / 1e9)
    del src, dst
    return best


def measure_bidir_peak(torch, dev) -> float:
    """Each-direction GB/s with H2D and D2H of 1 GiB running at once (partition's full-duplex roof)."""
    h_in = torch.empty(GIB, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(GIB, dtype=torch.uint8, pin_memory=True)
    d_in = torch.empty(GIB, dtype=torch.uint8, device=dev)
    d_out = torch.empty(GIB, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    best = 0.0
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(s1):
            for o in range(0, GIB, 256 * MIB):
                d_in[o:o + 256 * MIB].copy_(h_in[o:o + 256 * MIB], non_blocking=True)
        with torch.cuda.stream(s2):
            for o in range(0, GIB, 256 * MIB):
                h_out[o:o + 256 * MIB].copy_(d_out[o:o + 256 * MIB], non_blocking=True)
        torch.cuda.synchronize()
        best = max(best, GIB / (time.perf_counter() - t0) / 1e9)
    del h_in, h_out, d_in, d_out
    return best


# arithmetic type each workload's path computes in (bytes are moved as u8 everywhere)
DTYPE = {"grep": "u8", "wordcount": "u8 (u64 hashes, u64 counts)", "groupby": "u64 + f64",
         "groupby_sparse": "u64 + f64", "kmeans": "f32 distances, f64 sums", "partition": "u64", "kmer": "u64"}


def load_traffic() -> dict:
    """Per-unit traffic of the roofline kernels from one ncu --set full capture each (committed;
    the latest round's file wins per workload)."""
    out = {}
    for name in ("r01_traffic.json", "r02_traffic.json"):
        try:
            with open(os.path.join(ROOT, "profiles", name)) as f:
                out.update(json.load(f))
        except (OSError, ValueError):
            pass
    return out


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


# ------------------------------------------------------------------------------ host-side rooflines
def host_rooflines(args, shard, st, step_s: float, peak_h2d: float, tr, pack_rate=None) -> dict:
    """The two host-side resources a HYBRID step (CPU-packed + zero-copy chunks) is bound by,
    against peaks measured in this run (the C2 line must name its binding roofline):
      host_dram: bytes the host memory system moves per step / the live STREAM copy bandwidth (all
        cores). Per packed record: its offset (8 B, variable records) + every 64-B line its accessed
        extent touches (counted exactly from this shard's record addresses) + the packed bytes written
        (non-temporal) + the same bytes read by the DMA; per zero-copy record: its lines + its offset
        (DMA'd). Hardware prefetch may add lines, so this is a lower bound on the traffic.
      pcie_wire: H2D completion bytes per step / the DMA wire peak. Zero-copy keys cost the PCIe read
        bytes ncu measured per record (profiles/r01_traffic.json); DMAs carry their payload plus
        one 24-B TLP header+framing per 256-B max payload (x 280/256), and so does the peak."""
    import baselines
    hs = baselines.host_stream(2.0, 3)
    buf, off, n = shard["buf"], shard["off"], shard["n"]
    eo, E = (16, 32) if args.workload == "grep" else (0, 16)
    starts = (off.astype(np.uint64) if off is not None else np.arange(n, dtype=np.uint64) * np.uint64(shard["rec_size"]))
    a0 = starts + np.uint64(buf.ctypes.data + eo)
    lines = ((a0 + np.uint64(E - 1)) // np.uint64(64) - a0 // np.uint64(64) + np.uint64(1))
    lines_per_rec = float(lines.mean())
    rec_zc = st["records_zc"]
    rec_cpu = n - rec_zc
    off_b = 8 if off is not None else 0
    host_bytes = rec_cpu * (off_b + 64 * lines_per_rec + 2 * E) + rec_zc * (off_b + 64 * lines_per_rec)
    ach = host_bytes / step_s / 1e9
    zc_wire = tr["pcie_read_per_unit"] if tr and tr.get("unit") == "record" else None
    tlp = 280 / 256
    wire = (rec_zc * zc_wire if zc_wire else 0.0) + (st["bytes_h2d"] - st["bytes_zc"] + st["bytes_meta"]) * tlp
    wire_ach = wire / step_s / 1e9
    out = {}
    if pack_rate and st.get("ms_zc") and rec_zc:
        # The HYBRID step as a two-resource schedule: the link carries the zero-copy keys (bound by the
        # PCIe read-request rate: R_zc records/s, measured on the zero-copy gathers of this run's
        # profiled pass), the packed keys and every record's offset by DMA (payload peak BW), while the
        # host packs the rest at P records/s (measured alone in a CPU-assembly pass). With a share x of
        # records zero-copy: link(x) = a + b x, host(x) = c (1 - x); the best split balances them, and
        # T* = a + b x* is the least step time this host + link admit.
        r_zc = rec_zc / (st["ms_zc"] * 1e-3)
        a_ = (n * E + n * off_b) / (peak_h2d * 1e9)
        b_ = n / r_zc - n * E / (peak_h2d * 1e9)
        c_ = n / pack_rate
        x_opt = min(1.0, max(0.0, (c_ - a_) / (b_ + c_)))
        t_star = a_ + b_ * x_opt
        out["hybrid_schedule"] = {
            "bound": "link+host schedule", "t_bound_ms": round(t_star * 1e3, 3), "t_step_ms": round(step_s * 1e3, 3),
            "frac": t_star / step_s, "x_zc_opt": round(x_opt, 4), "x_zc_run": round(rec_zc / n, 4),
            "zc_records_per_s": r_zc, "pack_records_per_s": pack_rate, "dma_gbs": peak_h2d,
            "note": "frac = least admissible step time / measured step time (1.0 = at the bound)"}
    out.update({
        "host_dram": {"bound": "host_dram", "achieved": ach, "peak": hs["copy_gbs"], "unit": "GB/s",
                      "frac": ach / hs["copy_gbs"], "bytes_per_step": host_bytes,
                      "lines_per_record": round(lines_per_rec, 4), "records_cpu": rec_cpu, "records_zc": rec_zc,
                      "peak_source": f"STREAM copy (read + write bytes) on {hs['threads']} host threads, measured live "
                                     f"(read-only: {hs['read_gbs']:.1f} GB/s)"},
        "pcie_wire": {"bound": "pcie_wire", "achieved": wire_ach, "peak": peak_h2d * tlp, "unit": "GB/s",
                      "frac": wire_ach / (peak_h2d * tlp), "bytes_per_step": wire,
                      "zc_wire_bytes_per_record": zc_wire,
                      "peak_source": "pinned H2D DMA payload peak (live) x 280/256 TLP framing"},
    })
    return out


# ------------------------------------------------------------------------------ oracle timing
def oracle_sample(workload: str, shard: dict, target_s: float):
    """Time the oracle (as it stands) on a bounded prefix of the shard; returns (GB/s, sample str, s)."""
    import oracle
    buf, off = shard["buf"], shard["off"]

    def run(nrec):
        t0 = time.perf_counter()
        if workload == "grep":
            end = int(off[nrec]) if nrec < len(off) else len(buf)
            oracle.grep(buf[:end], off[:nrec], b"bigk")
        elif workload == "wordcount":
            end = int(off[nrec]) if nrec < len(off) else len(buf)
            oracle.wc(buf[:end], off[:nrec])
        elif workload in ("groupby", "groupby_sparse"):
            end = nrec * shard["rec_size"]
            oracle.groupby(buf[:end], nrec, shard["rec_size"], 4096)
        elif workload == "kmer":
            end = nrec * 256
            oracle.kmer(buf[:end], nrec, 31)
        elif workload == "partition":
            end = nrec * 16
            oracle.partition(buf[:end].view(np.uint64).reshape(-1, 2), 1024)
        else:
            end = nrec * 64
            oracle.kmeans(buf[:end].view(np.float32), shard["mu"])
        return time.perf_counter() - t0, end

    n = shard["n"]
    probe = max(1, min(n, n // 64))
    dt, nb = run(probe)
    want = min(n, max(probe, int(probe * target_s / max(dt, 1e-6))))
    dt, nb = run(want)
    return nb / dt / 1e9, f"first {want} of {n} records ({nb / GIB:.2f} GiB) of the rank-0 shard", dt


# ------------------------------------------------------------------------------ main arms
def main():
    global HUGE
    args = parse()
    HUGE = {"huge": True, "4k": False, "numpy": None}[args.pages]
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    gib = args.gib if args.gib is not None else WORKLOADS[args.workload][0]
    window = (args.window_mib or WORKLOADS[args.workload][1]) * MIB

    if args.impl == "reference":
        return reference_arm(args, rank, world, gib)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_mokhtaris14_b200 import bk

    # one process per GPU; BK_BENCH_BACKEND=gloo lets several ranks share one GPU for a smoke test
    backend = os.environ.get("BK_BENCH_BACKEND", "nccl")
    # BK_BENCH_DIST=1 runs the distributed path (process group, device-resident results, merge.py's
    # collectives) even at world size 1: `torchrun --nproc-per-node 1` exercises the real NCCL calls
    # on a one-GPU box (tests/test_gpu_nccl.py)
    dist_on = world > 1 or os.environ.get("BK_BENCH_DIST") == "1"
    local = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if dist_on:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    # ranks on one node share the host cores for CPU assembly (one pool per rank): bind each rank to
    # its GPU's NUMA-local share before the shard is generated (first touch) and the pool started
    if world > 1 and torch.cuda.device_count() > 1:
        cores = numa_local_cores(torch, local)
        if cores:
            os.sched_setaffinity(0, cores)
            if not args.host_threads:
                args.host_threads = len(cores)
    if not args.host_threads:
        args.host_threads = max(1, (os.cpu_count() or 1) // int(os.environ.get("LOCAL_WORLD_SIZE", "1")))
    shard = make_shard(args.workload, gib, rank, world, args.K)
    peak_h2d = measure_h2d_peak(torch, dev)
    peak_bidir = measure_bidir_peak(torch, dev) if args.workload == "partition" else None
    ctx = bk.Context(device=local, window_bytes=window, n_slots=args.slots, gather_mode=args.gather,
                     baseline_dbuf=args.impl == "dbuf", baseline_sbuf=args.impl == "sbuf",
                     host_threads=args.host_threads, lane_bytes=args.lane_bytes, zc_share_pm=args.zc_share,
                     profile=False, record_size=shard["rec_size"], keep_outputs_pinned=True)
    t0 = time.perf_counter()
    ctx.register(shard["buf"], shard["off"], n_records=shard["n"])
    reg_s = time.perf_counter() - t0
    stream = torch.cuda.current_stream()
    nbytes = len(shard["buf"])

    cap = max(shard["n"] // 50, 1 << 16)
    idx_out = np.empty(cap, np.uint64)
    # result arrays, allocated (and touched) once and reused by every step: host arrays at N=1 (the
    # caller reads its result on the host); at N>1 the aggregating kernels write device tensors that
    # the merge collectives reduce / gather in place (bk.h: result arrays may be device memory)
    kmer_out = wc_out = agg_out = None
    if args.workload == "kmer":
        kcap = 1 << 27
        kmer_out = ((torch.zeros(kcap, dtype=torch.int64, device=dev), torch.zeros(kcap, dtype=torch.int64, device=dev))
                    if dist_on else (np.zeros(kcap, np.uint64), np.zeros(kcap, np.uint64)))
    if args.workload == "wordcount":
        wcap = 1 << 20
        wc_out = ((torch.zeros(wcap, dtype=torch.int64, device=dev), torch.zeros(wcap, dtype=torch.int32, device=dev),
                   torch.zeros(wcap, dtype=torch.int64, device=dev), torch.zeros(wcap, dtype=torch.int64, device=dev),
                   torch.zeros(wcap, dtype=torch.int64, device=dev))
                  if dist_on else (np.zeros(wcap, np.uint64), np.zeros(wcap, np.uint32), np.zeros(wcap, np.uint64)))
    if args.workload in ("groupby", "groupby_sparse"):
        cq = torch.zeros(2, 4096, dtype=torch.int64, device=dev)
        agg_out = ((cq[0], cq[1], torch.zeros(4096, dtype=torch.float64, device=dev), cq) if dist_on else
                   (np.zeros(4096, np.uint64), np.zeros(4096, np.uint64), np.zeros(4096, np.float64)))
    if args.workload == "kmeans":
        agg_out = ((torch.zeros(args.K, dtype=torch.int64, device=dev),
                    torch.zeros(args.K, 16, dtype=torch.float64, device=dev))
                   if dist_on else (np.zeros(args.K, np.uint64), np.zeros((args.K, 16), np.float64)))

    from paper_conf_ipps_mokhtaris14_b200 import merge

    box = {}   # facts of the last step the roofline needs (k-mer windows)

    def one_step(ctx=ctx):
        """One pass of the whole hot path over this rank's shard, then the merge (N>1). Returns this
        rank's (merged) result, for --dump."""
        cs = stream.cuda_stream
        if args.workload == "grep":
            res = ctx.grep(b"bigk", first_index=shard["first"], stream=cs, out=idx_out)
            return {"idx": res, "place": merge.merge_grep_offsets(len(res)) if dist_on else (0, len(res))}
        if args.workload == "wordcount":
            r = ctx.wordcount(stream=cs, out=wc_out)
            if dist_on:   # all-gather of compacted {h1, h2, len, count, rank, off} rows, merged on the GPU
                rows = merge.merge_wordcount(ctx, *r)
                return {"rows": rows.cpu().numpy()}
            return {"off": r[0], "len": r[1], "count": r[2]}
        if args.workload == "kmer":
            km, ct, total = ctx.kmer(k=31, table_slots=1 << 28, stream=cs, out=kmer_out)
            box["kmer_windows"] = total
            if dist_on:
                rows = merge.merge_kmer(ctx, km, ct)
                return {"rows": rows.cpu().numpy()}
            return {"kmer": km, "count": ct}
        if args.workload == "partition":
            out, cc, bc = ctx.partition(1024, out=shard["out"], stream=cs)
            box["part_cc"] = cc
            if dist_on:
                start, boff = merge.merge_partition_offsets(bc)
                return {"start": start, "boff": boff, "cc": cc}
            return {"cc": cc, "bc": bc}
        if args.workload in ("groupby", "groupby_sparse"):
            c, q, a = ctx.groupby(4096, stream=cs, out=agg_out[:3])
            if dist_on:   # in place on the device buffers bk_run wrote
                merge.merge_sum(agg_out[3])
                merge.merge_sum(a)
                return {"count": c.cpu().numpy(), "qty": q.cpu().numpy(), "amount": a.cpu().numpy()}
            return {"count": c, "qty": q, "amount": a}
        c, s_, chk = ctx.kmeans(shard["mu"], first_index=shard["first"], stream=cs, out=agg_out)
        if dist_on:
            merge.merge_sum(c)
            merge.merge_sum(s_)
            chk = merge.merge_checksum(chk)
            return {"count": c.cpu().numpy(), "sum": s_.cpu().numpy(), "chk": chk}
        return {"count": c, "sum": s_, "chk": chk}

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    if dist_on:
        dist.barrier()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    wall, dev_ms, stats = [], [], []
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if dist_on:
            dist.barrier()
        for k in range(args.steps):
            h0 = time.perf_counter()
            ev[k][0].record(stream)
            one_step()
            ev[k][1].record(stream)
            ev[k][1].synchronize()
            wall.append(time.perf_counter() - h0)
            stats.append(ctx.stats())
        torch.cuda.synchronize()
        if dist_on:
            dist.barrier()
    dev_ms = [a.elapsed_time(b) for a, b in ev]
    t_dev = sum(dev_ms) / 1e3
    t_wall = sum(wall)
    if dist_on:  # max over ranks
        tt = torch.tensor([t_dev, t_wall], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_dev, t_wall = tt.tolist()
    if args.workload == "partition" and "part_cc" in box:
        # the optional bucket-major copy: a separately timed host pass, not in value
        dst = np.empty_like(shard["out"])
        dst.fill(0)   # fault the destination pages in first: a reused output buffer in steady state
        t0 = time.perf_counter()
        bk.partition_materialize(shard["out"], box["part_cc"], dst=dst)
        mt = time.perf_counter() - t0
        box["materialize"] = {"ms": round(mt * 1e3, 3), "gbs": round(dst.nbytes / mt / 1e9, 3),
                              "threads": os.cpu_count(),
                              "what": "bk_partition_materialize: chunk-major runs -> bucket-major stable order on "
                                      "the host (optional, timed separately, not part of value; destination pre-faulted)"}
        del dst
    st = dict(stats[-1])
    if args.dump:
        res = one_step()
        torch.cuda.synchronize()
        os.makedirs(args.dump, exist_ok=True)
        flat = {}
        for k, v in res.items():
            if hasattr(v, "cpu"):
                v = v.cpu().numpy()
            flat[k] = np.asarray(v)
        if args.workload == "partition":
            flat["out"] = shard["out"]
        np.savez(os.path.join(args.dump, f"rank{rank}.npz"), world=world, rank=rank, first=shard["first"],
                 n=shard["n"], **flat)
    if not args.no_profile:
        # per-stage CUDA events force eager issue (graph event nodes carry no timestamps), so the
        # stage breakdown comes from a separate profiled pass over the same shard
        pctx = bk.Context(device=local, window_bytes=window, n_slots=args.slots, gather_mode=args.gather,
                          baseline_dbuf=args.impl == "dbuf", baseline_sbuf=args.impl == "sbuf",
                          host_threads=args.host_threads, lane_bytes=args.lane_bytes, zc_share_pm=args.zc_share,
                          profile=True, record_size=shard["rec_size"], keep_outputs_pinned=True)
        pctx.register(shard["buf"], shard["off"], n_records=shard["n"])
        for _ in range(2):
            one_step(pctx)
        pst = pctx.stats()
        pctx.close()
        for k in ("ms_h2d", "ms_addrgen", "ms_gather", "ms_compute", "n_gather", "ms_cpu_gather", "ms_xfer_busy",
                  "ms_zc", "n_zc", "ms_relayout", "n_relayout", "n_chunks_zc", "bytes_zc", "records_zc", "ms_d2h", "n_d2h",
                  "ms_compute_busy", "ms_overlap", "fused_wait_frac", "fused_compute_frac", "fused_loader_wait_frac"):
            st[k] = pst[k]
        st["profiled_ms_device"] = pst["ms_device"]
    trace = None
    if not args.no_profile and not args.no_trace:
        # the timed pipeline itself (graph replay kept), every kernel and copy timed by CUPTI activity
        # records: the stage breakdown and overlap of the pass that matches ms_per_step
        try:
            tctx = bk.Context(device=local, window_bytes=window, n_slots=args.slots, gather_mode=args.gather,
                              baseline_dbuf=args.impl == "dbuf", baseline_sbuf=args.impl == "sbuf",
                              host_threads=args.host_threads, lane_bytes=args.lane_bytes, zc_share_pm=args.zc_share,
                              trace=True, record_size=shard["rec_size"], keep_outputs_pinned=True)
            tctx.register(shard["buf"], shard["off"], n_records=shard["n"])
            for _ in range(3):
                one_step(tctx)
            trace = tctx.stats()
            tctx.close()
        except bk.BkError as e:
            trace = {"unavailable": str(e)}
    total_bytes = nbytes * world * args.steps
    total_recs = shard["n"] * world * args.steps
    value = total_bytes / t_dev / 1e9
    link_bytes = (st["bytes_h2d"] + st["bytes_meta"]) * world * args.steps
    link_gbs = link_bytes / t_dev / 1e9

    # ---- roofline of the dominant stage (busy times from CUDA events on each stage's own stream)
    peaks = load_peaks()
    stage_ms = {"zc": st["ms_zc"], "relayout": st["ms_relayout"], "compute": st["ms_compute"],
                "addrgen": st["ms_addrgen"], "h2d": st["ms_h2d"]}
    # dominant stage: transfer (DMA / zero-copy gather) vs compute by the UNION of their busy
    # intervals (per-slot streams run kernels concurrently, so per-launch sums overcount); stage 1
    # (addrgen) runs a chunk ahead and is off the critical chain, so it is never the roofline kernel.
    # Inside the transfer side the zero-copy gathers and the copy-engine DMAs are told apart by their
    # own busy times; the HBM -> HBM interleave of DMA'd chunks is accounted separately (ms_relayout).
    if st.get("ms_compute_busy", 0.0) > st.get("ms_xfer_busy", 0.0):
        dom = "compute"
    else:
        dom = "zc" if st["n_chunks_zc"] and st["ms_zc"] >= st["ms_h2d"] else "h2d"
        if st.get("n_d2h") and st.get("ms_d2h", 0.0) > st[{"zc": "ms_zc", "h2d": "ms_h2d"}[dom]]:
            dom = "d2h"  # write-back (partition's bucket-sorted chunks) is the busier direction
    stage_ms["d2h"] = st.get("ms_d2h", 0.0)
    if st["gather_mode"] == 5:
        dom = "fused"   # word count as one persistent launch: stages 1-4 in k_wc_fused
    stage_ms["fused"] = st["ms_zc"]
    if dom == "fused":
        # the single launch pulls the text and the record offsets over PCIe (cp.async zero-copy into
        # its shared-memory ring) and computes on them: algorithmic bytes = text + offsets
        launches = max(st["n_zc"], 1)
        per_launch = st["bytes_h2d"] + st["bytes_meta"]
        roof = {"kernel": "k_wc_fused (stages 1-4, one persistent launch, zero-copy cp.async into shared memory)",
                "bound": "host_link", "peak": peak_h2d, "unit": "GB/s"}
    elif dom == "d2h":
        # copy-engine DMA of the per-chunk outputs back to the host, running full duplex with the
        # H2D stream: against the per-direction peak measured with both directions busy
        launches = max(st["n_d2h"], 1)
        per_launch = st["bytes_d2h"] / launches
        roof = {"kernel": "cudaMemcpyAsync D2H of per-chunk outputs (write-back, copy engine)", "bound": "host_link",
                "peak": peak_bidir if peak_bidir else peak_h2d, "unit": "GB/s"}
    elif dom == "h2d":
        # copy-engine DMA of packed (CPU) or raw (DENSE) chunks + offsets slices: host-link bound
        launches = max(st["n_chunks"] - st["n_chunks_zc"], 1)
        per_launch = (st["bytes_h2d"] - st["bytes_zc"] + st["bytes_meta"]) / launches
        roof = {"kernel": "cudaMemcpyAsync H2D of staged chunks (stage 3, copy engine)", "bound": "host_link",
                "peak": peak_h2d, "unit": "GB/s"}
    elif dom == "zc":
        # the zero-copy gather kernel (stages 2+3 fused): accessed bytes it pulled over PCIe per launch
        launches = max(st["n_zc"], 1)
        per_launch = st["bytes_zc"] / max(st["n_chunks_zc"], 1)
        roof = {"kernel": "k_gather_field/whole<zero-copy> (stages 2+3)", "bound": "host_link",
                "peak": peak_h2d, "unit": "GB/s"}
    else:
        launches = st["n_chunks"]
        # HBM-bound compute: reads the staged tiles (payload + padding)
        per_launch = (st["bytes_accessed"] + st["bytes_padding"]) / max(launches, 1)
        kname = f"{dom} ({args.workload})"
        if args.workload == "kmer" and box.get("kmer_windows"):
            # + the two-phase counting traffic per k-mer window: its 8-B hash appended to a coarse bin
            # (k_kmer_bin), read back and appended to its region's bucket (k_kmer_split), read once more
            # by the region's flush (k_kmer_flush): 32 B
            per_launch += 32 * box["kmer_windows"] / max(launches, 1)
            kname = "compute (kmer: k_kmer_bin + k_kmer_split + k_kmer_flush)"
        roof = {"kernel": kname, "bound": "hbm", "peak": peaks.get("hbm_gbs", 6650.0), "unit": "GB/s"}
    avg_ms = stage_ms[dom] / max(launches, 1)
    if avg_ms <= 0:  # --no-profile: no per-stage event times, so no per-launch figure
        avg_ms = float("nan")
    roof["achieved"] = per_launch / (avg_ms * 1e-3) / 1e9
    roof["peak_source"] = ("pinned H2D cudaMemcpyAsync measured live in this run (MEASURED_PEAKS.json has no "
                           "host-link entry)") if dom in ("h2d", "zc", "fused") else (
        "pinned H2D + D2H cudaMemcpyAsync running concurrently, per direction, measured live in this run"
        if dom == "d2h" else None) if roof["bound"] == "host_link" else (
        "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "fallback 6650 GB/s")
    roof["frac"] = roof["achieved"] / roof["peak"]
    roof["traffic"] = None
    tr = load_traffic().get(args.workload)
    if tr and tr.get("kernel", "").endswith("k_wc_fused") != (dom == "fused"):
        tr = None   # a capture of another kernel than this line's roofline kernel
    if tr and args.workload == "kmer":
        tr = None   # one capture is one of the three counting kernels, not the per-chunk compute
    if tr and dom == "fused":
        units = st["bytes_accessed"]
        roof["traffic"] = tr["traffic_per_unit"] * units
        roof["traffic_source"] = (f"{tr['what']} of {tr['kernel']}, ncu --set full ({tr['capture']}): "
                                  f"{tr['traffic_per_unit']:.3f} B per text byte x {units} bytes per launch; "
                                  f"algorithmic bytes per launch {per_launch:.0f} (text + offsets)")
    elif tr and ((dom == "zc" and tr["unit"] == "record") or (dom == "compute")):
        # bytes one launch moves, measured by ncu --set full on one launch of the same kernel
        # (profiles/r01_traffic.json, tools/gpu_traffic.sh), scaled to this run's units per launch
        if dom == "zc":
            units = st["records_zc"] / max(st["n_chunks_zc"], 1)
        elif tr["unit"] == "record":
            units = shard["n"] / max(st["n_chunks"], 1)
        else:
            units = st["bytes_accessed"] / max(st["n_chunks"], 1)
        roof["traffic"] = tr["traffic_per_unit"] * units
        roof["traffic_source"] = (f"{tr['what']} of {tr['kernel']}, ncu --set full ({tr['capture']}): "
                                  f"{tr['traffic_per_unit']:.2f} B per {tr['unit']} x {units:.0f} {tr['unit']}s "
                                  f"per launch; algorithmic bytes per launch {per_launch:.0f}" +
                                  ({"grep": "; a zero-copy read moves whole 32-B sectors (an 8-aligned 32-B key at +16 "
                                            "touches 1.75 of them on average) and every read completion carries PCIe TLP "
                                            "overhead, so the link traffic is ~2.7x the key bytes by construction, not "
                                            "re-reads",
                                    "groupby_sparse": "; each 16-B field is read as a whole 32-B sector of its 64-B "
                                                      "record plus PCIe TLP overhead per completion, ~4.4x the field "
                                                      "bytes by construction, not re-reads"}.get(args.workload, "")
                                   if dom == "zc" else ""))
    if dom == "zc" and args.workload == "grep":
        # the zero-copy key gather is PCIe read-request bound, not byte bound: one read request per
        # 128-B line a 32-B key touches (8-aligned keys: 1 + 3/16 = 1.1875 requests per record).
        # Peak = the request rate the phase-0 probe measured for one field per 256-B record
        # (profiles/r01_box_probe.txt: zc_sparse rec 256 -> 0.562 G records/s, one request each).
        recs_per_launch = st["records_zc"] / max(st["n_chunks_zc"], 1)
        req_rate = recs_per_launch * 1.1875 / (avg_ms * 1e-3)
        roof["request_rate"] = {"bound": "pcie_read_requests", "achieved": req_rate / 1e9, "peak": 0.562,
                                "unit": "G requests/s", "frac": req_rate / 0.562e9,
                                "peak_source": "profiles/r01_box_probe.txt zc_sparse (256-B stride, 1 request/record)"}
        roof["note"] = ("the zero-copy key gather is bound by outstanding PCIe read requests (one per 32-B key, "
                        "~84 B of read-completion traffic each), not by bytes: frac is against the H2D DMA byte "
                        "peak, request_rate.frac against the probed request-rate peak (DESIGN.md §6, §9)")
    if dom != "zc" and args.workload == "grep" and st.get("n_chunks_zc") and st.get("ms_zc"):
        # HYBRID with the packed chunks' DMA as the busiest stage: the zero-copy gather kernel (the
        # dominant KERNEL of the ncu launch list) still runs beside it, sharing the link; its own
        # per-launch rooflines, from the profiled pass
        zc_ms = st["ms_zc"] / st["n_chunks_zc"]
        recs = st["records_zc"] / st["n_chunks_zc"]
        key_gbs = recs * 32 / (zc_ms * 1e-3) / 1e9
        req = recs * 1.1875 / (zc_ms * 1e-3)
        roof["zc_gather"] = {"kernel": "k_gather_field<zero-copy> (stages 2+3)", "avg_launch_ms": zc_ms,
                             "launches_per_step": st["n_chunks_zc"], "achieved": key_gbs, "unit": "GB/s",
                             "frac": key_gbs / peak_h2d, "peak": peak_h2d,
                             "request_rate": {"bound": "pcie_read_requests", "achieved": req / 1e9, "peak": 0.562,
                                              "unit": "G requests/s", "frac": req / 0.562e9,
                                              "peak_source": "profiles/r01_box_probe.txt zc_sparse"},
                             "note": "runs concurrently with the DMAs of host-packed chunks (the two share the "
                                     "link), so both per-launch rates are below their solo rates; "
                                     "hybrid_schedule.frac is the step against the least time this host + link admit"}
    if dom == "fused":
        roof["fused"] = {"units": st["n_units"], "unit_bytes": st["unit_bytes"], "ctas": st["fused_grid"],
                         "loader_ctas": st["fused_loaders"], "ring_slots": st["fused_ring_slots"],
                         "consumer_wait_frac": round(st["fused_wait_frac"], 4),
                         "consumer_compute_frac": round(st["fused_compute_frac"], 4),
                         "loader_wait_frac": round(st["fused_loader_wait_frac"], 4),
                         "note": "in-kernel %globaltimer shares (profiled pass): consumers waiting for a unit's flag "
                                 "vs computing while loaders stream later units; loaders waiting for a free ring slot"}
    roof["avg_launch_ms"] = avg_ms
    roof["launches_per_step"] = launches
    if args.workload in ("grep", "groupby_sparse") and args.gather in ("auto", "hybrid") and args.impl == "ours" \
            and not args.no_profile:
        # the host packers alone (CPU assembly of every chunk, no zero-copy traffic): their rate. Every
        # rank runs the pass (one_step holds the merge collective), rank 0 reports
        cctx = bk.Context(device=local, window_bytes=window, n_slots=args.slots, gather_mode="cpu",
                          host_threads=args.host_threads, record_size=shard["rec_size"], keep_outputs_pinned=True)
        cctx.register(shard["buf"], shard["off"], n_records=shard["n"])
        one_step(cctx)
        one_step(cctx)
        cst = cctx.stats()
        cctx.close()
        pack_rate = shard["n"] / (cst["ms_cpu_gather"] * 1e-3) if cst["ms_cpu_gather"] else None
        if rank == 0 and st.get("n_chunks_cpu"):
            roof.update(host_rooflines(args, shard, st, t_dev / args.steps, peak_h2d, tr, pack_rate))

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(t_dev / args.steps * 1e3, 3),
        "step_ms": [round(x, 3) for x in dev_ms], "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": DTYPE[args.workload], "data": "synthetic (seeded counter RNG, gen/)",
        "config": {"workload": args.workload, "desc": WORKLOADS[args.workload][2],
                   "bytes_per_gpu": nbytes, "records_per_gpu": shard["n"], "window_bytes": window,
                   "n_slots": st["n_slots"],
                   "gather_mode": {1: "zc", 2: "cpu", 3: "dense", 4: "hybrid", 5: "fused", 6: "addr"}.get(st["gather_mode"], "?"),
                   "chunks_cpu_assembled": st["n_chunks_cpu"], "n_chunks": st["n_chunks"],
                   "lanes_per_chunk": st["lanes"], "chunk_budget_bytes": st["chunk_budget"],
                   "l2": "inputs (>=64 MiB per GPU, host-resident) exceed the 126 MB L2; streamed from host each step",
                   "plan_cache": "the chunk / lane / unit plan (a host O(n) pass over the record offsets, row a1) is "
                                 "computed by the first bk_run after registration (a warm-up step) and cached with the "
                                 "registration; timed steps reuse it (as they reuse the pinned registration)",
                   "parallelism": f"dp{world} (contiguous record shards, one PCIe link per GPU)",
                   **({"K": args.K} if args.workload == "kmeans" else {})},
        "records_per_s": total_recs / t_dev,
        "link_full_duplex": None if peak_bidir is None else {
            "peak_each_way_gbs": round(peak_bidir, 3), "achieved_each_way_gbs": round(link_gbs, 3),
            "frac": round(link_gbs / (peak_bidir * world), 4),
            "note": "partition streams n x 16 B in and the bucket-sorted n x 16 B back out concurrently"},
        "link": {"algorithmic_gbs": round(link_gbs, 3), "peak_h2d_gbs_per_gpu": round(peak_h2d, 3),
                 "frac": round(link_gbs / (peak_h2d * world), 4),
                 "bytes_per_step_per_gpu": st["bytes_h2d"] + st["bytes_meta"],
                 "payload_bytes": st["bytes_h2d"], "meta_bytes": st["bytes_meta"], "padding_bytes_hbm": st["bytes_padding"]},
        "stages_ms_per_step": {**{k: round(st[k], 3) for k in ("ms_h2d", "ms_addrgen", "ms_gather", "ms_zc",
                                                                "ms_relayout", "ms_compute", "ms_device",
                                                                "ms_cpu_gather", "ms_d2h")},
                               "n_zc": st["n_zc"], "n_relayout": st["n_relayout"],
                               "profiled_ms_device": round(st.get("profiled_ms_device", 0.0), 3),
                               "note": "per-stage busy sums from a profiled eager pass (CUDA events per stage "
                                       "per chunk); ms_device from the timed (graph-replayed when static) pass"},
        "timed_pass_trace": None if trace is None else ({"unavailable": trace["unavailable"]} if "unavailable" in trace else {
            "device_span_ms": round(trace["ms_trace_span"], 3), "records": trace["n_trace_records"],
            "span_vs_ms_per_step": round(trace["ms_trace_span"] / (t_dev / args.steps * 1e3), 4),
            "stages_ms": {k: round(trace[k], 3) for k in ("ms_h2d", "ms_addrgen", "ms_zc", "ms_relayout", "ms_compute",
                                                          "ms_d2h")},
            "launches": {"zc": trace["n_zc"], "relayout": trace["n_relayout"], "d2h": trace["n_d2h"]},
            "xfer_busy_ms": round(trace["ms_xfer_busy"], 3), "compute_busy_ms": round(trace["ms_compute_busy"], 3),
            "overlap_ms": round(trace["ms_overlap"], 3),
            "overlap_frac": round(trace["ms_overlap"] / max(min(trace["ms_xfer_busy"], trace["ms_compute_busy"]), 1e-9), 4),
            "link_busy_frac": round(trace["ms_xfer_busy"] / max(trace["ms_trace_span"], 1e-9), 4),
            "max_busy_frac": round(max(trace["ms_xfer_busy"], trace["ms_compute_busy"]) / max(trace["ms_trace_span"], 1e-9), 4),
            "how": "BK_FLAG_TRACE: CUPTI activity records of every kernel / copy of one graph-replayed (as timed) run; "
                   "transfer = H2D/D2H copies + zero-copy gathers (+ k_wc_fused, stages 1-4), compute = stage-4 "
                   "kernels; overlap_frac = |xfer n compute| / min(xfer, compute)"}),
        "overlap": {"xfer_busy_ms": round(st.get("ms_xfer_busy", 0.0), 3),
                    "compute_busy_ms": round(st.get("ms_compute_busy", 0.0), 3),
                    "overlap_ms": round(st.get("ms_overlap", 0.0), 3),
                    "overlap_frac": round(st.get("ms_overlap", 0.0) / max(min(st.get("ms_xfer_busy", 0.0),
                                                                              st.get("ms_compute_busy", 0.0)), 1e-9), 4),
                    "link_busy_frac": round(st.get("ms_xfer_busy", 0.0) / max(st.get("profiled_ms_device", 0.0), 1e-9), 4),
                    "max_busy_frac": round(max(st.get("ms_xfer_busy", 0.0), st.get("ms_compute_busy", 0.0)) /
                                           max(st.get("profiled_ms_device", 0.0), 1e-9), 4),
                    "how": "unions of per-chunk CUDA-event intervals of the transfer stages (DMA copies, zero-copy "
                           "gathers) and of the compute kernels, profiled pass; overlap_frac = |xfer n compute| / "
                           "min(xfer, compute); link_busy_frac = xfer union / device time; max_busy_frac = max(xfer, compute) "
                           "union / device time (SURVEY §8(d) overlap)"},
        "e2e": {"value": round(total_bytes / t_wall / 1e9, 3), "unit": "GB/s",
                "h2d_bytes_per_step": (st["bytes_h2d"] + st["bytes_meta"]) * world,
                "d2h_bytes_per_step": st["bytes_d2h"] * world,
                "note": "host wall clock around the public bk_run call (pinned host data in, results out to host); "
                        "it tracks the device-timed value because the data set never resides on the GPU: every "
                        "input byte of every step crosses the host link inside bk_run, in both measurements"},
        "roofline": roof,
        "gpu_launches": int(st["kernel_launches"]) * args.steps,
        # how the timed steps issued their device work (bk_stats.graph_issue of the last step)
        "graph_issue": {0: "eager", 1: "captured", 2: "replayed"}.get(int(st.get("graph_issue", 0)), "?"),
        "clocks": clk.summary(),
        "register_s": round(reg_s, 3),
        **({"materialize": box["materialize"]} if "materialize" in box else {}),
    }
    if args.impl != "ours":
        line["impl"] = args.impl
    if args.workload in ("grep", "groupby", "groupby_sparse", "kmeans", "wordcount") and not args.no_dbuf and \
            args.impl == "ours":
        # the paper's GPU double-buffering baseline (variant iv) on the same data, window and box
        dctx = bk.Context(device=local, window_bytes=window, baseline_dbuf=True, profile=False,
                          record_size=shard["rec_size"])
        dctx.register(shard["buf"], shard["off"], n_records=shard["n"])
        dsteps = max(1, min(args.steps, 20 if args.workload == "wordcount" else 3))   # WC steps are ~4 ms

        def dstep():
            if args.workload == "grep":
                dctx.grep(b"bigk", first_index=shard["first"], stream=stream.cuda_stream, out=idx_out)
            elif args.workload == "kmeans":
                dctx.kmeans(shard["mu"], first_index=shard["first"], stream=stream.cuda_stream)
            elif args.workload == "wordcount":
                dctx.wordcount(stream=stream.cuda_stream, out=wc_out)
            else:
                dctx.groupby(4096, stream=stream.cuda_stream)

        for _ in range(3 if args.workload == "wordcount" else 1):   # warm-up
            dstep()
        torch.cuda.synchronize()
        a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a_.record(stream)
        for _ in range(dsteps):
            dstep()
        b_.record(stream)
        b_.synchronize()
        dt = a_.elapsed_time(b_) / 1e3
        if dist_on:
            tt = torch.tensor([dt], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            dt = tt.item()
        dv = nbytes * world * dsteps / dt / 1e9
        line["baseline_dbuf"] = {"value": round(dv, 3), "unit": "GB/s", "steps": dsteps,
                                 "what": "cudaMemcpyAsync double buffering of whole-record chunks (2 x window/2, "
                                         "2 streams) + the same computation per thread-range (PAPER.md P:329-339, P:994-996)",
                                 "bigkernel_speedup": round(value / dv, 3)}
        dctx.close()
    if rank == 0 and not args.no_cpu_baseline and args.impl == "ours" and args.workload in (
            "grep", "groupby", "groupby_sparse", "kmeans", "partition", "kmer", "wordcount"):
        # the paper's multithreaded CPU variant (ii) on all host cores, same shard (kmeans: 1/16 sample,
        # k-mers: 1/4 sample)
        import baselines
        # all host cores (the variant-ii CPU baseline is the whole box's CPU), whatever OMP_NUM_THREADS
        # torchrun set and whatever NUMA-local affinity this rank's GPU pipeline runs under
        saved_aff = os.sched_getaffinity(0)
        try:
            os.sched_setaffinity(0, range(os.cpu_count() or 1))
        except OSError:
            pass
        baselines.set_threads(os.cpu_count() or 1)
        if args.workload == "wordcount":   # steady state: its per-thread tables persist across calls
            baselines.wordcount(shard["buf"], shard["off"])
        t0 = time.perf_counter()
        if args.workload == "grep":
            baselines.grep(shard["buf"], shard["off"])
            mt_bytes = nbytes
        elif args.workload == "kmeans":
            m = shard["n"] // 16
            baselines.kmeans(shard["buf"][: m * 64].view(np.float32).reshape(-1, 16), shard["mu"])
            mt_bytes = m * 64
        elif args.workload == "wordcount":
            baselines.wordcount(shard["buf"], shard["off"])
            mt_bytes = nbytes
        elif args.workload == "partition":
            baselines.partition(shard["buf"].view(np.uint64).reshape(-1, 2), 1024)
            mt_bytes = nbytes
        elif args.workload == "kmer":
            m = shard["n"] // 4   # a quarter of the reads, into the same 2^28-slot table size as the GPU's
            baselines.kmer(shard["buf"][: m * 256], m, k=31, slots=1 << 28)
            mt_bytes = m * 256
        else:
            baselines.groupby(shard["buf"], shard["n"], shard["rec_size"], 4096)
            mt_bytes = nbytes
        mt = mt_bytes / (time.perf_counter() - t0) / 1e9
        os.sched_setaffinity(0, saved_aff)
        line["cpu_mt_baseline"] = {"value": round(mt, 3), "unit": "GB/s", "cores": baselines.threads(),
                                   "what": "paper variant (ii): OpenMP over all host cores (baselines/cpu_mt.c)",
                                   "bigkernel_speedup": round(value / mt, 3)}
    if rank == 0 and not args.no_cpu_baseline:
        gbs, sample, secs = oracle_sample(args.workload, shard, 10.0)
        line["cpu_baseline"] = {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                                "sample": sample, "seconds": round(secs, 2)}
    if rank == 0:
        print(json.dumps(line), flush=True)
    ctx.close()
    if dist_on:
        dist.barrier()
        dist.destroy_process_group()


def reference_arm(args, rank, world, gib):
    """The oracle, as it stands, on this box's host cores: each step a bounded sample."""
    if rank != 0:
        return
    shard = make_shard(args.workload, gib, 0, 1)
    per_step_s = 4.0
    for _ in range(args.warmup):
        oracle_sample(args.workload, shard, 0.5)
    vals, secs = [], 0.0
    sample = ""
    for _ in range(args.steps):
        gbs, sample, s = oracle_sample(args.workload, shard, per_step_s)
        vals.append(gbs)
        secs += s
    v = statistics.mean(vals)
    line = {"metric": METRIC, "value": round(v, 4), "unit": "GB/s", "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": DTYPE[args.workload], "data": "synthetic (seeded counter RNG, gen/)",
            "config": {"workload": args.workload, "desc": WORKLOADS[args.workload][2],
                       "bytes_per_gpu": len(shard["buf"]), "records_per_gpu": shard["n"]},
            "ms_per_step": round(secs / args.steps * 1e3, 1),
            "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
