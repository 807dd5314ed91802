"""Summarise ncu outputs into profiles/ (run here, no GPU needed).

    python tools/ncu_summary.py gpurun_out/prof_vscale.ncu-rep ... > profiles/r01_kernels.md
    python tools/ncu_summary.py --launches gpurun_out/launches.csv > profiles/r01_launches.md
"""
import csv
import io
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__shared_mem_per_block_dynamic",
    "sm__cycles_elapsed.avg.per_second",
    "l1tex__t_bytes.sum",
    "lts__t_bytes.sum",
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [dict(zip(hdr, r)) for r in rows[2:]], dict(zip(hdr, units))


def tensor_keys(hdr):
    return [h for h in hdr if "tensor" in h and "pct" in h]


def summarise_rep(rep):
    recs, units = raw(rep)
    print(f"\n### {rep}\n")
    for r in recs:
        print(f"kernel `{r.get('Kernel Name', '?')}`\n")
        print("| metric | value | unit |\n|---|---|---|")
        keys = KEYS + [k for k in tensor_keys(r.keys()) if k not in KEYS]
        for k in keys:
            if k in r:
                print(f"| {k} | {r[k]} | {units.get(k, '')} |")
        print()


def summarise_launches(path):
    rows = list(csv.reader(open(path)))
    # ncu --csv --log-file: header line with "Kernel Name", "Metric Name", "Metric Value"
    start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[start]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    ui = hdr.index("Metric Unit") if "Metric Unit" in hdr else None
    tot = {}
    cnt = {}
    for r in rows[start + 1:]:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        v = float(r[vi].replace(",", ""))
        unit = r[ui] if ui is not None else "ns"
        ns = v * {"ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6, "nsecond": 1}.get(unit, 1)
        name = r[ki][:90]
        tot[name] = tot.get(name, 0) + ns
        cnt[name] = cnt.get(name, 0) + 1
    allns = sum(tot.values())
    print("| kernel | launches | total us | share |\n|---|---|---|---|")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"| `{k}` | {cnt[k]} | {v / 1e3:.1f} | {v / allns:.3f} |")


if __name__ == "__main__":
    if sys.argv[1] == "--launches":
        summarise_launches(sys.argv[2])
    else:
        for rep in sys.argv[1:]:
            summarise_rep(rep)
