#!/usr/bin/env python
"""Summarise ncu output (launch list CSV + `--set full` report) into a
markdown file under profiles/.  Runs here (no GPU needed to read reports).

    python scripts/summarize_ncu.py gpurun_out/r1_launch_list.csv gpurun_out/r1_full.ncu-rep profiles/r1_ncu.md \
        [F_H F_C [workload [config]]]

With F_H F_C it also merges the selective kernel's per-launch DRAM traffic and
L2->L1 read bytes into profiles/traffic.json under the workload's name (bench.py's
roofline.traffic and l2_view).
"""
import csv
import io
import subprocess
import sys
from collections import OrderedDict

METRICS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2->L1 read sectors"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 thru %"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM thru %"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__registers_per_thread", "regs"),
]


def launch_list(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = []
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            out.append((int(d["ID"]), d["Kernel Name"], d["Grid Size"], float(d["Metric Value"]) / 1e3))
    return out


def short(name):
    name = name.replace("pcgcn::<unnamed>::", "").replace("(anonymous namespace)::", "")
    return name.split("(")[0][:60]


def main(csv_path, rep_path, out_path):
    L = launch_list(csv_path)
    total = sum(t for _, _, _, t in L)
    agg = OrderedDict()
    for _, nm, grid, t in L:
        k = short(nm)
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += t
    lines = ["# ncu summary (one epoch, eager launches; cold-cache serialised times — compare SHARES)", "",
             f"source: `{csv_path}` ({len(L)} launches, {total / 1e3:.3f} ms total)", "",
             "| kernel | launches | total us | share |", "|---|---|---|---|"]
    for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"| `{k}` | {c} | {t:.1f} | {100 * t / total:.1f}% |")
    if rep_path:
        raw = subprocess.run(["ncu", "-i", rep_path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(raw)))
        if rows:
            hdr, units = rows[0], rows[1]
            lines += ["", f"## `--set full` capture: `{rep_path}`", "",
                      "| kernel | grid | " + " | ".join(lbl for _, lbl in METRICS) + " |",
                      "|---|---|" + "---|" * len(METRICS)]
            for d in rows[2:]:
                vals = []
                for m, _ in METRICS:
                    if m in hdr:
                        v, u = d[hdr.index(m)], units[hdr.index(m)]
                        vals.append(f"{v} {u}".strip())
                    else:
                        vals.append("-")
                lines.append(f"| `{short(d[hdr.index('Kernel Name')])}` | {d[hdr.index('Grid Size')]} | " +
                             " | ".join(vals) + " |")
    open(out_path, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))
    # per-launch DRAM traffic of the selective kernel for bench.py's roofline.traffic:
    # the capture's first sparse_agg launch is the layer-1 forward (F=H), the second the layer-2 one (F=C)
    if rep_path and len(sys.argv) > 5:
        import json
        import os
        fH, fC = int(sys.argv[4]), int(sys.argv[5])
        wl = sys.argv[6] if len(sys.argv) > 6 else "reddit"
        # the selective pass = segment kernel + row kernel; the capture holds the
        # layer-1 forward (F=H) launches first, then the layer-2 ones (F=C):
        # group by the lane layout template arguments <G, V, H> of the kernel name
        sp = [d for d in rows[2:] if "sparse_" in d[hdr.index("Kernel Name")]]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9,
                 "sector": 1, "Ksector": 1e3, "Msector": 1e6, "Gsector": 1e9}
        def g_of(d):
            nm = d[hdr.index("Kernel Name")]
            return ",".join(a.strip() for a in nm.rsplit("_kernel<", 1)[1].split(">", 1)[0].split(",")[:3])
        tr = {}
        groups = []
        for d in sp:
            if not groups or g_of(d) != g_of(groups[-1][0]):
                groups.append([])
            groups[-1].append(d)
        def one_call(grp):   # a call = [segment pass] + row pass; later calls of the same layout follow
            out = []
            for d in grp:
                out.append(d)
                if "sparse_row" in d[hdr.index("Kernel Name")]:
                    break
            return out
        groups = [one_call(g_) for g_ in groups]
        for key, grp in zip(("sparse_agg_F%d" % fH, "sparse_agg_F%d" % fC), groups[:2]):
            tot, l2 = 0.0, 0.0
            for d in grp:
                for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
                    tot += float(d[hdr.index(m)].replace(",", "")) * scale.get(units[hdr.index(m)], 1)
                m = "lts__t_sectors_srcunit_tex_op_read.sum"
                if m in hdr:
                    l2 += 32.0 * float(d[hdr.index(m)].replace(",", "")) * scale.get(units[hdr.index(m)], 1)
            tr[key] = int(tot)
            tr[key + "_l2_read_bytes"] = int(l2) if l2 else None
            # time-weighted L2 (LTS) throughput, % of its sustained peak (ncu's own roofline of the L2)
            tm = "gpu__time_duration.sum"
            for m, suffix in (("lts__throughput.avg.pct_of_peak_sustained_elapsed", "_lts_pct"),
                              ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "_dram_pct"),
                              ("l1tex__throughput.avg.pct_of_peak_sustained_active", "_l1tex_pct")):
                if m in hdr and tm in hdr:
                    ts = [float(d[hdr.index(tm)].replace(",", "")) for d in grp]
                    ps = [float(d[hdr.index(m)].replace(",", "")) for d in grp]
                    tr[key + suffix] = round(sum(t * p for t, p in zip(ts, ps)) / max(sum(ts), 1e-30), 2)
            tr[key + "_kernels"] = [short(d[hdr.index("Kernel Name")]) for d in grp]
        tr["source"] = rep_path
        if len(sys.argv) > 7:
            tr["config"] = sys.argv[7]   # the plan options / θ the capture ran with (bench.py checks it)
        tp = os.path.join(os.path.dirname(out_path), "traffic.json")
        allt = json.load(open(tp)) if os.path.exists(tp) else {}
        allt[wl] = tr
        json.dump(allt, open(tp, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 and sys.argv[2] != "-" else None, sys.argv[3])
