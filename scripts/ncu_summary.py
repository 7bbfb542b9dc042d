"""Compact per-launch summary of an ncu report: ncu_summary.py report.ncu-rep"""
import csv, io, subprocess, sys

WANT = [("gpu__time_duration.sum", "us"), ("dram__bytes_read.sum", "MB_rd"), ("dram__bytes_write.sum", "MB_wr"),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm%"),
        ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "mem%"),
        ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2%"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor%"),
        ("launch__grid_size", "grid"), ("launch__registers_per_thread", "regs")]
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, units = rows[0], rows[1]
print("| kernel | " + " | ".join(w[1] for w in WANT) + " |")
print("|---" * (len(WANT) + 1) + "|")
for r in rows[2:]:
    d = dict(zip(hdr, r))
    name = d.get("Kernel Name", "?").split("(")[0].split("::")[-1]
    vals = []
    for key, _ in WANT:
        v = d.get(key, "")
        u = units[hdr.index(key)] if key in hdr else ""
        try:
            x = float(v.replace(",", ""))
            if key == "gpu__time_duration.sum":
                x = x * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u, 1)
            if key.startswith("dram__bytes"):
                x = x * {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3}.get(u, 1)
            vals.append(f"{x:.1f}")
        except ValueError:
            vals.append(v or "-")
    print(f"| {name} | " + " | ".join(vals) + " |")
