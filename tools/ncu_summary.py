"""Summaries of ncu output for profiles/ (run here, on the CPU box).

  python tools/ncu_summary.py launches <launches.csv>      per-kernel launch count, time, share
  python tools/ncu_summary.py full <report.ncu-rep> ...     key metrics per captured launch
  python tools/ncu_summary.py traffic <report.ncu-rep> <config> <kernel> [json]
                                                           dram bytes per launch -> profiles/ncu_traffic.json
"""
from __future__ import annotations

import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

FULL_METRICS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram%"),
    ("lts__t_sector_hit_rate.pct", "L2hit%"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2thr%"),
    ("l1tex__t_sector_hit_rate.pct", "L1hit%"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps%"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "lanes/inst"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "ld_sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "ld_requests"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem_wavefronts"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed", "smem%"),
    ("smsp__inst_executed.sum", "warp_inst"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
]

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0,
         "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9}


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    agg = defaultdict(lambda: [0, 0.0])
    for d in data:
        k = d["Kernel Name"].split("(")[0].strip()
        agg[k][0] += 1
        agg[k][1] += float(d["Metric Value"]) * SCALE.get(d["Metric Unit"], 1e-9)
    tot = sum(v[1] for v in agg.values())
    out = ["| kernel | launches | total ms | ms/launch | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"| `{k}` | {v[0]} | {v[1] * 1e3:.3f} | {v[1] * 1e3 / v[0]:.4f} | {v[1] / tot * 100:.1f}% |")
    out.append(f"| total | {sum(v[0] for v in agg.values())} | {tot * 1e3:.3f} | | 100% |")
    return "\n".join(out)


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {}
        for name, short in FULL_METRICS:
            if name in hdr:
                i = hdr.index(name)
                try:
                    d[short] = float(r[i].replace(",", "")) * SCALE.get(units[i], 1)
                except ValueError:
                    d[short] = r[i]
        d["kernel"] = r[hdr.index("Kernel Name")].split("(")[0] if "Kernel Name" in hdr else "?"
        res.append(d)
    return res


def full(reps):
    out = ["| report | kernel | time ms | DRAM rd MB | DRAM wr MB | DRAM GB/s | DRAM % | L2 hit % | L2 thr % | L1 hit % | SM % | warps % | regs | grid |",
           "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in reps:
        for d in raw(rep):
            t = d.get("time", 0) or 1e-30
            gbs = (d.get("dram_rd", 0) + d.get("dram_wr", 0)) / t / 1e9
            out.append(f"| {rep.split('/')[-1]} | `{d['kernel']}` | {t * 1e3:.3f} | {d.get('dram_rd', 0) / 1e6:.1f} | "
                       f"{d.get('dram_wr', 0) / 1e6:.1f} | {gbs:.0f} | {d.get('dram%', 0):.1f} | {d.get('L2hit%', 0):.1f} | "
                       f"{d.get('L2thr%', 0):.1f} | {d.get('L1hit%', 0):.1f} | {d.get('SM%', 0):.1f} | "
                       f"{d.get('warps%', 0):.1f} | {d.get('regs', '')} | {d.get('grid', '')} |")
    out += ["", "| report | kernel | lanes / inst | ld sectors / request | smem wavefronts (M) | smem % | warp inst (M) |",
            "|---|---|---|---|---|---|---|"]
    for rep in reps:
        for d in raw(rep):
            spr = d.get("ld_sectors", 0) / d["ld_requests"] if d.get("ld_requests") else 0
            out.append(f"| {rep.split('/')[-1]} | `{d['kernel']}` | {d.get('lanes/inst', 0):.1f} | {spr:.2f} | "
                       f"{d.get('smem_wavefronts', 0) / 1e6:.1f} | {d.get('smem%', 0):.1f} | {d.get('warp_inst', 0) / 1e6:.1f} |")
    return "\n".join(out)


def traffic(rep, config, kernel, path="profiles/ncu_traffic.json"):
    ds = raw(rep)
    per = [d.get("dram_rd", 0) + d.get("dram_wr", 0) for d in ds]
    try:
        j = json.load(open(path))
    except Exception:
        j = {}
    j.setdefault(config, {})[kernel] = {"dram_bytes_per_launch": sum(per) / len(per), "launches": len(per),
                                        "source": rep.split("/")[-1],
                                        "note": "ncu --set full, dram__bytes_read.sum + dram__bytes_write.sum, mean over captured launches"}
    json.dump(j, open(path, "w"), indent=1)
    return j


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(launches(sys.argv[2]))
    elif sys.argv[1] == "full":
        print(full(sys.argv[2:]))
    elif sys.argv[1] == "traffic":
        print(json.dumps(traffic(*sys.argv[2:]), indent=1))
