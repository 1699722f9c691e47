"""Top CUDA source lines of an ncu report by warp-stall samples (needs -lineinfo and
--import-source on at capture time).

    python tools/ncu_src.py gpurun_out/prof.ncu-rep [top]
"""
import csv
import io
import os
import subprocess
import sys


def main(rep, top=30, filt=()):
    out = subprocess.run(["ncu", "-i", rep, *filt, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname = "?"
    hdr = None
    lines = []
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = os.path.basename(r[1])
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or not r[0]:
            continue
        try:
            s = int(r[4] or 0)
            ins = int(r[7] or 0)
        except (ValueError, IndexError):
            continue
        lines.append((s, ins, f"{fname}:{r[0]}", r[1].strip()))
    tot = sum(x[0] for x in lines) or 1
    print(f"total samples {tot}")
    for s, ins, where, src in sorted(lines, reverse=True)[:top]:
        print(f"{100 * s / tot:5.1f}% {s:6d} {ins:9d} {where:18s} {src[:90]}")


if __name__ == "__main__":
    # optional 3rd+ args: ncu import filters, e.g. -k regex:bk_voxels --launch-skip 0 --launch-count 1
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30, tuple(sys.argv[3:]))
