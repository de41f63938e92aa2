"""Print the key ncu metrics + top stall reasons of every kernel in a .ncu-rep.
usage: python tools/ncu_summary.py gpurun_out/prof_x.ncu-rep"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "smsp__inst_executed.sum", "lts__t_sectors_srcunit_tex_aperture_sysmem.sum"]


def main(path, nstall=6):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(h, r))
        print(f"== {d['Kernel Name'][:70]}  (ID {d['ID']})")
        for k in KEYS:
            if k in d:
                print(f"   {k:70s} {d[k]:>14s} {units[h.index(k)]}")
        st = []
        for k in h:
            if k.startswith("smsp__average_warps_issue_stalled") and k.endswith("per_issue_active.ratio"):
                try:
                    st.append((float(d[k].replace(",", "")), k))
                except ValueError:
                    pass
        st.sort(reverse=True)
        print("   stalls/issue: " + ", ".join(
            f"{k.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')}={v:.1f}"
            for v, k in st[:int(nstall)]))


if __name__ == "__main__":
    main(*sys.argv[1:])
