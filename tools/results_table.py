"""Markdown rows of DESIGN.md §12's results table from bench.py JSON lines.
python tools/results_table.py profiles/r01_bench_all.jsonl"""
import json
import sys

DESC = {
    "C2": "**C2** R=1M, 625K-op batches, 10/10/80 (default; the paper's Table 5.1 workload)",
    "C1": "C1 R=10K, 6250-op batches, 10/10/80",
    "C2-100": "C2-100 Contains-only, full 1M structure, 10M-op batch",
    "C2-2020": "C2-2020 [20,20,60], 312.5K-op batches",
    "C2-5050": "C2-5050 [50,50,0], 125K-op batches",
    "C3": "C3 R=10M, 6.25M-op batches, 10/10/80",
    "C3-zipf": "C3 Zipf(0.99), mutating keys without replacement (R2)",
    "C3-zipf-raw": "C3 raw Zipf(0.99), combining mode (R26)",
    "C2-zipf-raw": "C2 raw Zipf(0.99), combining mode (R26)",
    "C4-16": "C4-16 100M keys, Contains-only, 50M-op batches",
    "C4-32": "C4-32 same, the paper's 256-B chunks",
    "M1-1-98": "[1,1,98] (M1-1-98)",
    "M5-5-90": "[5,5,90] (M5-5-90)",
    "M20-20-60-10M": "[20,20,60] R = 10M, 625K-op batches",
    "INS-1M": "Insert-only, R ops from empty (INS-1M, Fig 5.4b)",
    "DEL-1M": "Delete-only, R ops from full (DEL-1M, Fig 5.4c)",
    "C5": "**C5** R=1B, 500M live keys, 125M-op batches (8 timed), one GPU",
    "C5-S2": "C5-S2: one shard of C5 at 2 GPUs (R=500M, 250M keys, 62.5M-op batches), its local work",
    "C5-S4": "C5-S4: one shard of C5 at 4 GPUs (R=250M, 125M keys, 31.25M-op batches), its local work",
    "C5-S8": "C5-S8: one shard of C5 at 8 GPUs (R=125M, 62.5M keys, 15.6M-op batches), its local work",
}


def row(d):
    c = d["config"]
    w = c["workload"]
    p = d.get("phase_ms_per_step", {})
    srch = p.get("search", 0.0)
    r = (d.get("roofline_kernels") or {}).get("search") or d.get("roofline") or {}
    e2e = d.get("e2e") or {}
    cpu = d.get("cpu_baseline") or {}
    runs = d.get("runs") or {}
    ci = runs.get("ci95_half_width")
    v = f"{d['value']:.0f}" + (f" ± {ci:.0f}" if ci is not None else "")
    v = f"**{v}**" if w in ("C2", "C5") else v
    roof = f"{r.get('bound', '-')} {r.get('frac', 0):.2f}" if r else "-"
    rg = (r.get("random_gathers") or {}).get("frac")
    if rg is not None:
        roof += f" (gathers {rg:.2f} of R_rand)"
    return (f"| {DESC.get(w, w)} | {c.get('chunk_entries', '')} | {v} | {e2e.get('value', 0):.0f} | "
            f"{srch:.3f} / {p.get('update', 0):.3f} / {p.get('upkeep_rebuild', 0):.3f} | "
            f"{d.get('chunk_reads_per_contains', 0):.2f} | {roof} | {cpu.get('value', 0):.1f} |")


def main():
    lines = [json.loads(x) for x in open(sys.argv[1]) if x.strip().startswith("{")]
    by = {d["config"]["workload"]: d for d in lines if "config" in d and "workload" in d["config"]}
    for w in DESC:
        if w in by:
            print(row(by[w]))


if __name__ == "__main__":
    main()
