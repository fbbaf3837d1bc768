"""Summaries of ncu captures for profiles/ (committed evidence).

    python tools/ncu_summary.py ROUND LAUNCHES.csv FULL.ncu-rep [CONFIG_NAME]

Writes profiles/rNN_launches.md (per-kernel device time of the launch list,
cold-cache and serialised: compare shares, not absolutes),
profiles/rNN_engine_ncu.md (headline metrics of the `--set full` capture of
the engine kernel plus the top stall locations) and updates
profiles/ncu_traffic.json (DRAM bytes per launch of the dominant kernel,
read by bench.py for roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe active"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput"),
    ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "memory throughput"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy"),
    ("lts__t_bytes.sum", "L2 traffic (all requests)"),
    ("l1tex__m_xbar2l1tex_read_bytes.sum", "L2 -> SM read bytes"),
    ("lts__t_sectors_srcunit_ltcfabric.sum", "L2 sectors from the other die (fabric)"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def ncu(*args):
    return subprocess.run(["ncu", *args], capture_output=True, text=True, check=True).stdout


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[hi], rows[hi + 1:]
    ik, iv = hdr.index("Kernel Name"), hdr.index("Metric Value")
    per = collections.defaultdict(list)
    ours = re.compile(r"\b(eng|ew|tc|simt)::")   # the library's kernels (not torch's input generation)
    for r in data:
        if not ours.search(r[ik]):
            continue
        per[r[ik].split("(")[0]].append(float(r[iv].replace(",", "")) / 1e3)   # ns -> us
    return per


def raw_metrics(rep):
    rows = list(csv.reader(io.StringIO(ncu("-i", rep, "--page", "raw", "--csv"))))
    h, u, v = rows[0], rows[1], rows[2]
    out = {}
    for name, label in METRICS:
        if name in h:
            i = h.index(name)
            out[name] = (label, v[i], u[i])
    return out


def top_stalls(rep, n=15):
    rows = list(csv.reader(io.StringIO(ncu("-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"))))
    f, line, hdr, agg = None, None, None, collections.Counter()
    for r in rows:
        if r and r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if not hdr or len(r) < 6:
            continue
        if r[2] == "-":
            line = (f, r[0], r[1].strip()[:90])
            continue
        if r[0] == "" and r[2].startswith("0x") and line:
            try:
                agg[line] += float(r[4] or 0)
            except ValueError:
                pass
    tot = sum(agg.values()) or 1.0
    return [(100 * v / tot, k) for k, v in agg.most_common(n)]


def main():
    rnd, lcsv, rep = sys.argv[1], sys.argv[2], sys.argv[3]
    cfg = sys.argv[4] if len(sys.argv) > 4 else "bert_base_stack"
    os.makedirs(PROF, exist_ok=True)
    per = launches(lcsv)
    tot = sum(sum(v) for v in per.values())
    with open(os.path.join(PROF, f"r{rnd}_launches.md"), "w") as fo:
        fo.write(f"# Round {rnd}: launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`)\n\n")
        fo.write("Cold-cache, serialised per-launch times of every kernel of ours in the captured\n"
                 "bench.py run (k-search off); compare SHARES with the live bench numbers.\n\n")
        fo.write("| kernel | launches | total us | avg us | share |\n|---|---|---|---|---|\n")
        for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
            fo.write(f"| `{k}` | {len(v)} | {sum(v):.1f} | {sum(v) / len(v):.1f} | {sum(v) / tot:.1%} |\n")
    m = raw_metrics(rep)
    stalls = top_stalls(rep)
    with open(os.path.join(PROF, f"r{rnd}_engine_ncu.md"), "w") as fo:
        fo.write(f"# Round {rnd}: `ncu --set full` of one fused engine step ({cfg})\n\n")
        fo.write("| metric | value |\n|---|---|\n")
        for name, (label, val, unit) in m.items():
            fo.write(f"| {label} (`{name}`) | {val} {unit} |\n")
        fo.write("\nTop warp-stall locations (all samples, % of kernel):\n\n| % | file:line | source |\n|---|---|---|\n")
        for pct, (f, ln, src) in stalls:
            fo.write(f"| {pct:.1f} | {f}:{ln} | `{src.replace('|', '/')}` |\n")
    rd = float(m["dram__bytes_read.sum"][1]) if "dram__bytes_read.sum" in m else 0.0
    wr = float(m["dram__bytes_write.sum"][1]) if "dram__bytes_write.sum" in m else 0.0
    unit = m.get("dram__bytes_read.sum", ("", "", "byte"))[2]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
    tp = os.path.join(PROF, "ncu_traffic.json")
    traffic = json.load(open(tp)) if os.path.exists(tp) else {}
    traffic.setdefault(cfg, {})["engine_step"] = (rd + wr) * scale
    json.dump(traffic, open(tp, "w"), indent=1)
    print("wrote", PROF)


if __name__ == "__main__":
    main()
