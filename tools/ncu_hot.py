"""Top SASS lines by warp-stall samples from an ncu report's source page.
usage: python tools/ncu_hot.py report.ncu-rep [kernel_regex] [top]"""
import csv
import io
import subprocess
import sys


def main(path, kre=None, top=25):
    cmd = ["ncu", "-i", path, "--page", "source", "--csv"]
    if kre:
        cmd += ["--kernel-name", f"regex:{kre}"]
    raw = subprocess.run(cmd, capture_output=True, text=True).stdout
    lines = raw.splitlines()
    # one or more kernels: split on the "Kernel Name" header lines
    blocks, cur = [], []
    for ln in lines:
        if ln.startswith('"Kernel Name"'):
            if cur:
                blocks.append(cur)
            cur = [ln]
        else:
            cur.append(ln)
    if cur:
        blocks.append(cur)
    for b in blocks[:2]:
        print(b[0][:120])
        rows = list(csv.reader(io.StringIO("\n".join(b[1:]))))
        h = rows[0]
        si = h.index("Warp Stall Sampling (All Samples)")
        src = h.index("Source")
        tot = sum(int(r[si] or 0) for r in rows[1:] if len(r) > si)
        best = sorted(rows[1:], key=lambda r: -int(r[si] or 0) if len(r) > si else 0)[:int(top)]
        for r in best:
            print(f"{int(r[si]):6d} {100 * int(r[si]) / max(tot, 1):5.1f}%  {r[0][-6:]}  {r[src].strip()[:90]}")


if __name__ == "__main__":
    main(*sys.argv[1:])
