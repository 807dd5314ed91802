"""One markdown row per profiled launch (run here, no GPU needed):

    python tools/ncu_compact.py gpurun_out/prof_*.ncu-rep > profiles/r02_kernels.md
"""
import csv
import io
import subprocess
import sys

COLS = [("gpu__time_duration.sum", "us"), ("dram__bytes_read.sum", "DRAM read"),
        ("dram__bytes_write.sum", "DRAM write"),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % peak"),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM % peak"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe %"),
        ("launch__registers_per_thread", "regs"), ("launch__grid_size", "grid")]


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(c for c, _ in COLS)],
                         capture_output=True, text=True).stdout
    lines = [l for l in out.splitlines() if l.startswith('"')]
    rd = list(csv.reader(io.StringIO("\n".join(lines))))
    head, units, data = rd[0], rd[1], rd[2:]
    for r in data:
        d = dict(zip(head, r))
        u = dict(zip(head, units))
        yield d, u


def main():
    print("| report | kernel | " + " | ".join(n for _, n in COLS) + " |")
    print("|---|---|" + "---|" * len(COLS))
    for rep in sys.argv[1:]:
        for d, u in rows(rep):
            vals = []
            for c, _ in COLS:
                v = d.get(c, "")
                unit = u.get(c, "")
                vals.append(f"{v} {unit}".strip() if unit and unit not in ("%",) and c.startswith("dram__bytes") else v)
            print(f"| {rep.split('/')[-1]} | `{d.get('Kernel Name', '')}` | " + " | ".join(vals) + " |")


if __name__ == "__main__":
    main()
