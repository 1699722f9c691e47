"""Attribute an ncu capture's per-SASS-instruction counts to CUDA source lines.

    python tools/ncu_lines.py <report.ncu-rep> <mangled kernel name> [libam.so] [top] [block index]

Needs the .so that was profiled (line info from -lineinfo): its SASS offsets
are matched with the report's SASS page.  Prints instructions executed and
warp-stall samples per innermost source line and per kernel-level line (the
outermost call site of inlined code), so a phase of a fused kernel can be
costed.  Runs here (no GPU).
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LOC = re.compile(r'"([^"]+)", line (\d+)')


def sass_lines(so, func):
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(so)], cwd=tmp, capture_output=True)
    cub = [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")]
    out = {}
    for c in cub:
        dis = subprocess.run(["nvdisasm", "-g", "-gi", c], capture_output=True, text=True).stdout
        start = dis.find(f".text.{func}:")
        if start < 0:
            continue
        end = dis.find("\n.text.", start + 10)
        body = dis[start:end if end > 0 else len(dis)]
        inner = outer = None
        fresh = True  # the first comment after an instruction carries the full inline chain
        for ln in body.splitlines():
            s = ln.strip()
            if s.startswith("//## File"):
                locs = LOC.findall(s)
                if locs and fresh:
                    inner = (os.path.basename(locs[0][0]), int(locs[0][1]))
                    outer = (os.path.basename(locs[-1][0]), int(locs[-1][1]))
                fresh = False
                continue
            fresh = True
            m = re.match(r"/\*([0-9a-f]{4,})\*/", s)
            if m:
                out[int(m.group(1), 16)] = (inner, outer)
    return out


def main():
    rep, func = sys.argv[1], sys.argv[2]
    so = sys.argv[3] if len(sys.argv) > 3 else os.path.join(ROOT, "paper_conf_icpp_chenktkv19_b200", "libam.so")
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    # one block per kernel: a "Kernel Name" row, then a header row
    blocks, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            blocks.append(cur)
        elif cur is not None:
            cur["rows"].append(r)
    lines = sass_lines(so, func)
    srcs = {}
    if len(sys.argv) > 5:  # only the kernel block(s) of this index in the report (the one `func` names)
        blocks = [blocks[int(i)] for i in sys.argv[5].split(",")]
    for b in blocks:
        hdr = b["rows"][0]
        ix = {k: i for i, k in enumerate(hdr)}
        data = b["rows"][1:]
        base = int(data[0][ix["Address"]], 16)
        per_in = collections.Counter()
        per_out = collections.Counter()
        st_in = collections.Counter()
        st_out = collections.Counter()
        tot_i = tot_s = 0
        for r in data:
            off = int(r[ix["Address"]], 16) - base
            ins = int(r[ix["Instructions Executed"]] or 0)
            stl = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
            tot_i += ins
            tot_s += stl
            inner, outer = lines.get(off, (None, None))
            per_in[inner] += ins
            per_out[outer] += ins
            st_in[inner] += stl
            st_out[outer] += stl
        print(f"# {b['name']}: {tot_i} warp instructions, {tot_s} stall samples")

        def src(loc):
            if loc is None:
                return ""
            if loc[0] not in srcs:
                p = os.path.join(ROOT, "paper_conf_icpp_chenktkv19_b200", "csrc", loc[0])
                srcs[loc[0]] = open(p).read().splitlines() if os.path.exists(p) else []
            L = srcs[loc[0]]
            return L[loc[1] - 1].strip()[:70] if 0 < loc[1] <= len(L) else ""

        for title, ci, cs in (("kernel-level line (outermost call site)", per_out, st_out),
                              ("innermost line", per_in, st_in)):
            print(f"\n## by {title}: instr% stall% location source")
            keys = sorted(set(ci) | set(cs), key=lambda k: -(cs[k] / max(tot_s, 1) + ci[k] / max(tot_i, 1)))
            for k in keys[:top]:
                name = f"{k[0]}:{k[1]}" if k else "?"
                print(f"{100 * ci[k] / max(tot_i, 1):6.2f} {100 * cs[k] / max(tot_s, 1):6.2f}  {name:18s} {src(k)}")


if __name__ == "__main__":
    main()
