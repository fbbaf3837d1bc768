"""Per-kernel evidence table from an ncu --csv metrics capture (one row per
launch x metric): launches, mean duration, DRAM bytes per launch and the
achieved DRAM GB/s, tensor-pipe active %.  python tools/ncu_kernels.py CSV OUT.md TITLE"""
import collections
import csv
import sys

M_T = "gpu__time_duration.sum"
M_R = "dram__bytes_read.sum"
M_W = "dram__bytes_write.sum"
M_TC = "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"
M_DP = "dram__throughput.avg.pct_of_peak_sustained_elapsed"
SCALE = {"ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "nsecond": 1e-9, "msecond": 1e-3, "byte": 1, "Kbyte": 1e3,
         "Mbyte": 1e6, "Gbyte": 1e9, "%": 1}


def main():
    path, out, title = sys.argv[1], sys.argv[2], sys.argv[3]
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    iid, ik, im, iu, iv = (h.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    per = collections.defaultdict(lambda: collections.defaultdict(dict))
    for r in rows[hi + 1:]:
        name = r[ik].split("(")[0].replace("void ", "")
        if not any(t in name for t in ("eng::", "ew::", "tc::", "simt::")):
            continue
        v = float(r[iv].replace(",", "")) * SCALE.get(r[iu], 1)
        per[name][r[iid]][r[im]] = v
    lines = [f"# {title}", "", "| kernel | launches | mean us | DRAM MB / launch | DRAM GB/s | DRAM % of peak "
             "| tensor pipe active % |", "|---|---|---|---|---|---|---|"]
    for name, launches in sorted(per.items(), key=lambda kv: -sum(x.get(M_T, 0) for x in kv[1].values())):
        L = list(launches.values())
        t = sum(x.get(M_T, 0) for x in L) / len(L)
        by = sum(x.get(M_R, 0) + x.get(M_W, 0) for x in L) / len(L)
        dp = sum(x.get(M_DP, 0) for x in L) / len(L)
        tc = sum(x.get(M_TC, 0) for x in L) / len(L)
        lines.append(f"| `{name}` | {len(L)} | {t * 1e6:.1f} | {by / 1e6:.2f} | {by / t / 1e9 if t else 0:.0f} | "
                     f"{dp:.1f} | {tc:.1f} |")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
