"""Summarise an ncu capture + launch list into profiles/ (run here, no GPU needed).

    python tools/summarize_ncu.py <tag> [config] [maps per captured launch]
reads gpurun_out/prof_<tag>.ncu-rep and gpurun_out/launches_<tag>.csv, writes
profiles/<tag>_launches.txt, profiles/<tag>_<kernel>_ncu.txt and merges each captured
kernel's DRAM bytes into profiles/ncu_summary.json (by_config[config][kernel]), which bench.py reads
for `traffic` and `warp_inst_per_launch`.
"""
import csv
import io
import json
import os
import subprocess
import re
import sys
from collections import OrderedDict, defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def base_name(k):
    """'void am::am_pipeline_kernel<(bool)1>(am::FusedParams)' -> 'am_pipeline_kernel'."""
    k = re.sub(r"<.*>", "", k.split("(")[0] if "<" not in k.split("(")[0] else k[:k.index("<")])
    return k.replace("void ", "").split("::")[-1].strip()


_STAGES = {"bk_cones": ("l0_cones", "l1_cones", "live_cones"), "bk_rows": ("l0_rows", "l1_rows", "live_rows")}
_PLAIN = {"am_latency_kernel": "fused_pipeline", "bk_init": "init", "bk_level0": "level0", "bk_level1": "level1",
          "bk_stream": "stream", "bk_map": "clear_map", "bk_bricks": "bricks", "bk_bricks_fused": "bricks", "bk_voxels": "voxels", "bk_band": "band",
          "am_pipeline_kernel": "fused_pipeline", "filter_kernel": "filter", "baseline_kernel": "baseline",
          "clear_map_kernel": "clear_map", "band_exact_kernel": "band", "brick_test_kernel": "bricks",
          "brick_voxels_kernel": "voxels"}


def stage_name(full):
    """Kernel name as am_kernel_name() reports it (AM_K_* of include/am.h), or the base name."""
    b = base_name(full)
    if b in _STAGES:
        m = re.search(r"<\(int\)(\d)>|<(\d)>", full)
        if m:
            return _STAGES[b][int(m.group(1) or m.group(2))]
    return _PLAIN.get(b, b)


def ncu_csv(rep, page):
    out = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main():
    tag = sys.argv[1]
    config = sys.argv[2] if len(sys.argv) > 2 else "C3"
    maps = int(sys.argv[3]) if len(sys.argv) > 3 else 1  # AMs computed by the captured launch
    prof = os.environ.get("PROF_DIR") or os.path.join(ROOT, "profiles")  # (on the GPU box: under gpurun_out/)
    os.makedirs(prof, exist_ok=True)
    lc = os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv")
    if os.path.exists(lc):
        rows = list(csv.reader(open(lc)))
        start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
        hdr = rows[start]
        ix = {k: j for j, k in enumerate(hdr)}
        per = defaultdict(list)
        seq = []
        for r in rows[start + 1:]:
            if len(r) < len(hdr):
                continue
            name = stage_name(r[ix["Kernel Name"]])
            v = float(r[ix["Metric Value"]].replace(",", ""))
            per[name].append(v)
            seq.append((name, r[ix["Grid Size"]], v))
        with open(os.path.join(prof, f"{tag}_launches.txt"), "w") as f:
            f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none (cold, serialised): {config}\n")
            f.write("# per kernel: launches, mean ns, share of the listed time\n")
            tot = sum(sum(v) for v in per.values())
            for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
                f.write(f"{k:40s} {len(v):5d} {sum(v) / len(v):12.0f} {100 * sum(v) / tot:6.1f}%\n")
            f.write("\n# launch sequence (first 24)\n")
            for name, g, v in seq[:24]:
                f.write(f"{name:40s} {g:16s} {v:10.0f} ns\n")
    rep = os.path.join(ROOT, "gpurun_out", f"prof_{tag}.ncu-rep")
    if not os.path.exists(rep):
        return
    det = ncu_csv(rep, "details")
    h = det[0]
    kernels = OrderedDict()
    for r in det[1:]:
        d = dict(zip(h, r))
        key = (d["ID"], stage_name(d["Kernel Name"]))
        kernels.setdefault(key, []).append((d["Section Name"], d["Metric Name"], d["Metric Value"], d["Metric Unit"]))
    raw = ncu_csv(rep, "raw")
    rh, ru = raw[0], raw[1]
    for kidx, ((kid, kname), mets) in enumerate(kernels.items()):
        rawrow = dict(zip(rh, raw[2 + kidx])) if len(raw) > 2 + kidx else {}
        rawu = dict(zip(rh, ru))
        keep = ["Duration", "DRAM Throughput", "Memory Throughput", "Compute (SM) Throughput", "Executed Ipc Active",
                "Issue Slots Busy", "Registers Per Thread", "Achieved Occupancy", "Theoretical Occupancy",
                "Executed Instructions", "L2 Hit Rate", "L1/TEX Hit Rate", "Eligible Warps Per Scheduler",
                "No Eligible", "Avg. Active Threads Per Warp", "Grid Size", "Block Size",
                "Dynamic Shared Memory Per Block"]
        with open(os.path.join(prof, f"{tag}_{kname}_{kid}_ncu.txt"), "w") as f:
            f.write(f"# ncu --set full --clock-control none: {kname} (launch id {kid}), {config}\n")
            for sec, name, val, unit in mets:
                if name in keep:
                    f.write(f"{name:34s} {val:>16s} {unit}\n")
            for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
                      "sm__inst_executed.sum", "launch__registers_per_thread"):
                if k in rawrow:
                    f.write(f"{k:34s} {rawrow[k]:>16s} {rawu.get(k, '')}\n")
        if "dram__bytes_read.sum" in rawrow:
            def tobytes(v, u):
                v = float(v.replace(",", ""))
                return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            rd = tobytes(rawrow["dram__bytes_read.sum"], rawu["dram__bytes_read.sum"])
            wr = tobytes(rawrow["dram__bytes_write.sum"], rawu["dram__bytes_write.sum"])
            sp = os.path.join(prof, "ncu_summary.json")
            try:
                summ = json.load(open(sp))
            except Exception:
                summ = {}
            ent = {"config": config, "tag": tag, "maps_per_launch": maps,
                   "dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
                   "source": f"gpurun_out/prof_{tag}.ncu-rep (ncu --set full), launch id {kid}"}
            for sec, name, val, unit in mets:
                if name == "Executed Instructions" and unit == "inst":
                    ent["warp_inst_per_launch"] = float(val.replace(",", ""))
            if "gpu__time_duration.sum" in rawrow:
                ent["ncu_duration_us"] = tobytes(rawrow["gpu__time_duration.sum"], "") / (
                    1e3 if rawu.get("gpu__time_duration.sum") == "nsecond" else 1)
            old = summ.get("by_config", {}).get(config, {}).get(kname)
            if old and old.get("tag") == tag:  # same stage captured twice (clear_map): average
                for k2 in ("dram_bytes_per_launch", "dram_read", "dram_write", "warp_inst_per_launch",
                           "ncu_duration_us"):
                    if k2 in ent and k2 in old:
                        n_ = old.get("launches_averaged", 1)
                        ent[k2] = (old[k2] * n_ + ent[k2]) / (n_ + 1)
                ent["launches_averaged"] = old.get("launches_averaged", 1) + 1
            summ.setdefault("by_config", {}).setdefault(config, {})[kname] = ent
            if config == "C3":  # (the default workload's entries also under "kernels")
                summ.setdefault("kernels", {})[kname] = ent
            json.dump({"kernels": summ.get("kernels", {}), "by_config": summ["by_config"]}, open(sp, "w"), indent=1)

if __name__ == "__main__":
    main()
