"""Oracle wall-clock per AM on the host cores (SURVEY.md 8(d) "wall-clock per AM, with a 1-thread time
on C1 and C2 for a per-core figure"): full fp64 oracle maps (the definition, with its exact-safe
shortcuts, voxels in model order -- the oracle as it stands) with 1 thread and with every core.
    python tools/oracle_timing.py [C1 C2 ...]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import scenes  # noqa: E402


def main(names):
    print(f"host: {os.cpu_count()} logical CPUs", flush=True)
    for name in names:
        cfg = scenes.CONFIGS[name]
        C, H = cfg.leaves()
        p = cfg.pivots(1)[0]
        tests = float(len(H)) * cfg.m * cfg.n
        for nt in (1, os.cpu_count() or 1):  # (explicit: a thread count set by one call persists in OpenMP)
            t0 = time.perf_counter()
            st, used = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n, nthreads=nt, return_threads=True)
            dt = time.perf_counter() - t0
            print(f"{name} ({len(H)} voxels, {cfg.m}x{cfg.n}): {used} thread(s): {dt:.2f} s per AM, "
                  f"{tests / dt:.3g} voxel-orientation tests/s ({tests / dt / used:.3g} per thread); "
                  f"clear {int((st == 0).sum())}, band {int((st == 1).sum())}, blocked {int((st == 2).sum())}",
                  flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C1", "C2"])
