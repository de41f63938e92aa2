"""Fold ncu --metrics captures of k_gather (tools/ncu_r02h.sh) into profiles/traffic.json and
print a summary: per-launch DRAM, sysmem-read and PCIe-read bytes and the duration.
usage: python tools/traffic_from_ncu.py <tag> CONFIG:ALPHA ..."""
import csv
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def per_launch(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    d = {}
    for r in rows[hi + 1:]:
        d.setdefault(r[0], {})[r[h.index("Metric Name")]] = float(r[h.index("Metric Value")].replace(",", ""))
    return list(d.values())


def main(tag, *keys):
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    tj = json.load(open(tp))
    for key in keys:
        cfg, alpha = key.split(":")
        path = os.path.join(ROOT, "gpurun_out", f"hostlink_{cfg}_{alpha}_{tag}.csv")
        L = per_launch(path)
        m = lambda k: statistics.mean(x[k] for x in L)  # noqa: E731
        ent = {"dram_bytes": m("dram__bytes_read.sum") + m("dram__bytes_write.sum"),
               "dram_read_bytes": m("dram__bytes_read.sum"),
               "dram_write_bytes": m("dram__bytes_write.sum"),
               "sysmem_read_bytes": 32 * m("syslts__t_sectors_aperture_sysmem_op_read.sum"),
               "pcie_read_bytes": m("pcie__read_bytes.sum"),
               "ncu_duration_ms": m("gpu__time_duration.sum") / 1e6, "launches": len(L),
               "host_gather": 0}
        tj[f"{cfg}:{float(alpha)}"] = ent
        print(f"{cfg} alpha {alpha}: {len(L)} launches, {ent['ncu_duration_ms']:.3f} ms, DRAM read "
              f"{ent['dram_read_bytes'] / 1e6:.1f} MB + write {ent['dram_write_bytes'] / 1e6:.1f} MB, "
              f"sysmem read {ent['sysmem_read_bytes'] / 1e6:.1f} MB, PCIe read {ent['pcie_read_bytes'] / 1e6:.1f} MB")
    tj["_source"] += f"; {', '.join(keys)} -- profiles/{tag}_traffic.txt (tools/ncu_{tag}.sh)"
    json.dump(tj, open(tp, "w"), indent=1)


if __name__ == "__main__":
    main(*sys.argv[1:])
