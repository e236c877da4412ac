"""Per-kernel share of a bench step from an ncu launch list (gpu__time_duration.sum CSV).

python tools/launch_summary.py launches.csv
A step = the launches between two L2 flushes (the 256-MiB FillFunctor bench.py runs
between timed steps); the last `--steps` such steps are the timed ones.  ncu serialises
launches and runs them cold, so absolute times differ from the bench's CUDA events; the
SHARE of each kernel in a step is what must agree (B200_PROFILING.md)."""
import argparse
import collections
import csv


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--steps", type=int, default=4)
    a = ap.parse_args()
    rows = [r for r in csv.reader(open(a.csv)) if len(r) > 10]
    h, rows = rows[0], rows[1:]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    seq = [(r[ki].split("(")[0].replace("void ", "").replace("gfsl_dev::", ""),
            float(r[vi].replace(",", "")) / 1e3) for r in rows]
    steps, cur = [], None
    for name, t in seq:
        # the L2 flush before a timed step: torch's 256-MiB zero_ (FillFunctor in older
        # torch, a vectorized elementwise kernel in newer), ~70 us
        if (("FillFunctor" in name) or name.startswith("native::vectorized_elementwise")) and t > 20:
            if cur:
                steps.append(cur)
            cur = []
            continue
        if cur is not None:
            targs = name[name.find("<") + 1:name.rfind(">")].split(",") if "<" in name else []
            if "search_kernel" in name and len(targs) >= 3 and targs[2].strip() == "1":  # counting replay
                steps.append(cur)
                cur = None
                continue
            if not name.startswith("native::"):
                cur.append((name, t))
    if cur:
        steps.append(cur)
    steps = steps[-a.steps:]
    tot = collections.defaultdict(float)
    cnt = collections.defaultdict(int)
    for st in steps:
        for name, t in st:
            tot[name] += t
            cnt[name] += 1
    step_us = sum(tot.values()) / len(steps)
    print(f"{len(steps)} steps from {a.csv}; mean step = {step_us:.1f} us of serialised kernel time")
    print(f"{'kernel':48s} {'launches/step':>13s} {'us/step':>9s} {'share':>7s}")
    for name in sorted(tot, key=lambda n: -tot[n]):
        print(f"{name[:48]:48s} {cnt[name] / len(steps):13.2f} {tot[name] / len(steps):9.1f} {tot[name] / len(steps) / step_us:7.1%}")


if __name__ == "__main__":
    main()
