"""DRAM traffic of the TMA copy kernel per algorithmic byte, from one ncu capture of bench.py.

Usage: python tools/ncu_traffic.py <ncu metrics csv> <DYO_COPY_LOG file> > profiles/ncu_traffic.json

The csv is `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
-k regex:copy_records --csv` of a bench run with DYO_COPY_LOG set; launch i of the capture is line i
of the log (both in host launch order). Algorithmic bytes of a D2D copy launch = 2 x bytes moved
(read + write). bench.py scales its live per-launch algorithmic bytes by the measured ratio.
"""
import collections
import csv
import json
import sys

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "ns": 1e-3, "usecond": 1,
         "us": 1, "msecond": 1e3, "ms": 1e3}


def main(path_csv, path_log):
    rows = list(csv.reader(open(path_csv)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ii, ki, mi, ni, ui = (h.index("ID"), h.index("Kernel Name"), h.index("Metric Name"),
                          h.index("Metric Value"), h.index("Metric Unit"))
    per = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if not r[ki].startswith("copy_records_tma_kernel"):
            continue
        v = float(r[ni].replace(",", "")) * SCALE.get(r[ui], 1)
        per.setdefault(int(r[ii]), {})[r[mi]] = v
    logged = [int(x) for x in open(path_log).read().split()]
    launches = list(per.values())
    n = min(len(launches), len(logged))
    alg = sum(2 * b for b in logged[:n])
    dram = sum(l["dram__bytes_read.sum"] + l["dram__bytes_write.sum"] for l in launches[:n])
    us = sum(l["gpu__time_duration.sum"] for l in launches[:n])
    out = {"copy_records_tma_kernel": {
        "launches": n, "alg_bytes": alg, "dram_bytes": dram, "dram_per_alg_byte": round(dram / alg, 4),
        "serialised_gbs": round(alg / (us * 1e-6) / 1e9, 1),
        "source": "ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                  "--clock-control none -k regex:copy_records of python bench.py --steps 2 --warmup 1 "
                  "(MoE), paired with DYO_COPY_LOG"}}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
