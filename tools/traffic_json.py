#!/usr/bin/env python3
"""Per-unit memory / link traffic of each bench line's roofline kernel, from one ncu --set full
capture per kernel (tools/gpu_traffic.sh) plus the bench JSON line of the same command (units per
launch). Writes profiles/r02_traffic.json; bench.py scales it to its own launch size into
roofline.traffic.

    python tools/traffic_json.py r02h > profiles/r02_traffic.json
"""
import csv
import io
import json
import subprocess
import sys

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
         "byte/s": 1, "Kbyte/s": 1e3, "Mbyte/s": 1e6, "Gbyte/s": 1e9, "Tbyte/s": 1e12}


def raw(rep: str) -> dict:
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, r = rows[0], rows[1], rows[2]

    def val(m):
        i = hdr.index(m)
        return float(r[i].replace(",", "")) * SCALE.get(units[i], 1.0)

    return {"kernel": r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "").replace("unnamed>::", ""),
            "t": val("gpu__time_duration.sum"),
            "dram": val("dram__bytes_read.sum") + val("dram__bytes_write.sum"),
            "pcie_rd": val("pcie__read_bytes.sum.per_second") * val("gpu__time_duration.sum")}


def main(tag: str) -> None:
    res = {}
    for w, unit in (("grep", "record"), ("groupby_sparse", "record"), ("wordcount", "byte"), ("kmer", "record")):
        rep = f"gpurun_out/{tag}_tr_{w}.ncu-rep"
        try:
            k = raw(rep)
            line = next(json.loads(x) for x in open(f"gpurun_out/{tag}_tr_{w}.json") if x.startswith('{"metric"'))
        except Exception as e:  # noqa: BLE001 - report which capture is missing
            print(f"skip {w}: {e}", file=sys.stderr)
            continue
        # launches per step: one per chunk, except the fused word count (one persistent launch)
        chunks = 1 if line["config"].get("gather_mode") == "fused" else line["config"]["n_chunks"]
        units = (line["config"]["records_per_gpu"] if unit == "record" else line["config"]["bytes_per_gpu"]) / chunks
        link = w in ("grep", "groupby_sparse", "wordcount")  # zero-copy reads: the bound is the host link
        res[w] = {
            "kernel": k["kernel"], "capture": rep, "launch_ms": k["t"] * 1e3, "unit": unit,
            "units_per_launch": units,
            "what": ("PCIe read bytes (pcie__read_bytes.sum.per_second x gpu__time_duration.sum): the "
                     "link traffic of the zero-copy gather" if link else
                     "dram__bytes_read.sum + dram__bytes_write.sum"),
            "traffic_per_unit": (k["pcie_rd"] if link else k["dram"]) / units,
            "dram_per_unit": k["dram"] / units,
            "pcie_read_per_unit": k["pcie_rd"] / units,
            "note": ("one launch from the middle of the run, average units per launch of that run (ragged last "
                     "chunk aside); ncu replays the kernel with caches flushed between passes, so DRAM bytes "
                     "are cold-cache figures (an upper bound for kernels whose tables live in L2)"),
        }
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01x")
