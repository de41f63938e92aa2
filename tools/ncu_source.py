"""Warp-stall samples per CUDA source line of one kernel launch in an .ncu-rep
(cuda+sass source view: SASS rows are attributed to the preceding CUDA line).
usage: python tools/ncu_source.py rep.ncu-rep kernel_regex [launch_skip] [top_n]"""
import csv
import io
import subprocess
import sys


def main(path, kregex=".", skip="0", top="25"):
    cmd = ["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass",
           "--kernel-name", f"regex:{kregex}", "--launch-skip", skip, "--launch-count", "1"]
    raw = subprocess.run(cmd, capture_output=True, text=True).stdout
    fname, h, agg, cur = "?", None, {}, None
    for r in csv.reader(io.StringIO(raw)):
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].rsplit("/", 1)[-1]
            continue
        if r[0] == "Line No":
            h = r
            continue
        if h is None or len(r) < 7:
            continue
        if r[0]:  # a CUDA source line
            cur = (fname, r[0], r[1].strip()[:100])
            continue
        try:
            n = int(r[h.index("Warp Stall Sampling (All Samples)")])
        except (ValueError, IndexError):
            continue
        if cur:
            agg[cur] = agg.get(cur, 0) + n
    tot = sum(agg.values()) or 1
    for (f, ln, src), n in sorted(agg.items(), key=lambda x: -x[1])[: int(top)]:
        print(f"{100 * n / tot:5.1f}%  {f}:{ln:<5} {src}")


if __name__ == "__main__":
    main(*sys.argv[1:])
