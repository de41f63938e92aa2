"""Summarise a round's ncu captures into profiles/ (tracked):
  profiles/<tag>_launches.csv      -- the raw ncu launch list of the bench command
  profiles/<tag>_launch_summary.txt -- per-kernel totals and shares (one step = 1 batch)
  profiles/<tag>_ncu_<kernel>.txt  -- key metrics + stalls of each --set full capture
  profiles/traffic.json            -- DRAM bytes per k_gather launch (bench roofline 'traffic')
usage: python tools/make_profiles.py <tag>"""
import contextlib
import csv
import io
import json
import os
import shutil
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import launches as L  # noqa: E402
import ncu_summary as S  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(tag):
    src = os.path.join(ROOT, "gpurun_out")
    dst = os.path.join(ROOT, "profiles")
    os.makedirs(dst, exist_ok=True)
    shutil.copy(os.path.join(src, f"launches_{tag}.csv"), os.path.join(dst, f"{tag}_launches.csv"))
    buf = io.StringIO()
    with contextlib.redirect_stdout(buf):
        print(f"# ncu launch list of `python bench.py --steps 10 --warmup 3 --no-sweep "
              f"--no-cpu-baseline` (PR, alpha=1, default pipeline depth), --cache-control none --clock-control none;")
        print("# per-launch times are serialised by ncu: compare SHARES with the bench, not absolutes")
        print("## all launches (includes load/presample/build_cache/shuffle setup)")
        L.main(os.path.join(src, f"launches_{tag}.csv"))
        print("## last 70 launches (= the last 10 steps, the bench's e2e loop: seed, 2x(khop, compact), "
              "fixup, gather)")
        L.main(os.path.join(src, f"launches_{tag}.csv"), 70)
    open(os.path.join(dst, f"{tag}_launch_summary.txt"), "w").write(buf.getvalue())
    traffic = {}
    for k in ["k_gather", "k_compact", "k_khop", "k_seed_init", "k_fixup"]:
        rep = os.path.join(src, f"prof_{k}_{tag}.ncu-rep")
        if not os.path.exists(rep):
            continue
        buf = io.StringIO()
        with contextlib.redirect_stdout(buf):
            print(f"# ncu --set full --clock-control none --cache-control none, bench config (PR, alpha=1)")
            S.main(rep, 8)
        open(os.path.join(dst, f"{tag}_ncu_{k}.txt"), "w").write(buf.getvalue())
        if k == "k_gather":
            raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                                 text=True).stdout
            rows = list(csv.reader(io.StringIO(raw)))
            h = rows[0]
            vals = []
            for r in rows[2:]:
                d = dict(zip(h, r))
                unit_r = rows[1][h.index("dram__bytes_read.sum")]
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[unit_r]
                unit_w = rows[1][h.index("dram__bytes_write.sum")]
                scale_w = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[unit_w]
                vals.append(float(d["dram__bytes_read.sum"].replace(",", "")) * scale +
                            float(d["dram__bytes_write.sum"].replace(",", "")) * scale_w)
            traffic["PR:1.0"] = sum(vals) / len(vals)
    if traffic:
        json.dump({**traffic, "_source": f"profiles/{tag}_ncu_k_gather.txt (dram read+write bytes "
                   "per k_gather launch, ncu --set full)"},
                  open(os.path.join(dst, "traffic.json"), "w"), indent=1)
    print(open(os.path.join(dst, f"{tag}_launch_summary.txt")).read())


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01")
