"""Key metrics of an ncu report (raw page), unit-normalised: bytes, microseconds, percent.
python tools/ncu_metrics.py report.ncu-rep"""
import csv
import io
import json
import subprocess
import sys

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3,
         "second": 1e6, "s": 1e6, "%": 1, "": 1,
         "register/thread": 1, "inst": 1}
WANT = {"time_us": "gpu__time_duration.sum", "dram_read": "dram__bytes_read.sum",
        "dram_write": "dram__bytes_write.sum", "lts_bytes": "lts__t_bytes.sum",
        "l2_hit_pct": "lts__t_sector_hit_rate.pct", "l1_hit_pct": "l1tex__t_sector_hit_rate.pct",
        "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1_data_pipe_pct": "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "dram_throughput_pct": "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
        "registers": "launch__registers_per_thread", "inst_executed": "smsp__inst_executed.sum"}


def metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[h.index("Kernel Name")].split("(")[0]}
        for k, n in WANT.items():
            if n not in h:
                d[k] = None
                continue
            i = h.index(n)
            try:
                d[k] = float(r[i].replace(",", "")) * SCALE.get(units[i], 1)
            except ValueError:
                d[k] = None
        res.append(d)
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(json.dumps({"report": p, "kernels": metrics(p)}, indent=1))
