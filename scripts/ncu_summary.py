"""Summarise ncu captures for profiles/ (run here, on the CPU box, on files brought back by gpurun).

  python scripts/ncu_summary.py --rep gpurun_out/prof_jit_c5.ncu-rep --launches gpurun_out/launches.csv \
      --name round1_c5_jit --config c5 --out profiles/

Writes profiles/<name>.md (key SOL / pipe / stall metrics per profiled launch and the launch list
with each kernel's share of the step) and merges the DRAM bytes per launch into
profiles/ncu_summary.json (read by bench.py for roofline.traffic).
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput % of peak"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU pipe active % of peak"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe active % of peak"),
    ("sm__inst_executed_pipe_alu.sum", "warp instructions on the ALU pipe"),
    ("sm__inst_executed_pipe_fma.sum", "warp instructions on the FMA pipe"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy %"),
    ("sm__inst_executed.avg.per_cycle_active", "IPC (per SM, active)"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__block_size", "block size"),
    ("launch__grid_size", "grid size"),
    ("dram__bytes_read.sum", "DRAM bytes read"),
    ("dram__bytes_write.sum", "DRAM bytes written"),
    ("sm__cycles_active.avg", "SM active cycles"),
    ("sm__cycles_elapsed.avg", "SM elapsed cycles"),
]


def raw_rows(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep", action="append", default=[])
    ap.add_argument("--launches")
    ap.add_argument("--name", required=True)
    ap.add_argument("--config", default="c5")
    ap.add_argument("--out", default="profiles")
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    os.makedirs(a.out, exist_ok=True)
    md = [f"# ncu summary — {a.name}", ""]
    if a.note:
        md += [a.note, ""]
    dram_per_launch = []
    alu_pct, dur_ns = [], []
    for rep in a.rep:
        hdr, units, rows = raw_rows(rep)
        idx = {n: i for i, n in enumerate(hdr)}
        md += [f"## `{os.path.basename(rep)}` (ncu --set full --clock-control none)", ""]
        for r in rows:
            md.append(f"### launch {r[idx['ID']]}: `{r[idx['Kernel Name']][:60]}`")
            md.append("")
            md.append("| metric | value | unit |")
            md.append("|---|---|---|")
            for k, label in KEYS:
                if k in idx:
                    md.append(f"| {label} (`{k}`) | {r[idx[k]]} | {units[idx[k]]} |")
            stalls = []
            for n, i in idx.items():
                if "issue_stalled" in n and n.endswith("per_issue_active.ratio"):
                    try:
                        v = float(r[i])
                    except ValueError:
                        continue
                    if v >= 0.05:
                        stalls.append((v, n))
            md.append("")
            md.append("Warp stall reasons (cycles per issued instruction, >= 0.05): " +
                      ", ".join(f"{n.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')} {v:.2f}"
                                for v, n in sorted(stalls, reverse=True)))
            md.append("")
            scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            for key, acc in (("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", alu_pct),
                             ("gpu__time_duration.sum", dur_ns)):
                try:
                    acc.append(float(r[idx[key]]) * ({"ms": 1e6, "us": 1e3, "usecond": 1e3, "msecond": 1e6}.get(units[idx[key]], 1.0)
                                                     if key == "gpu__time_duration.sum" else 1.0))
                except (KeyError, ValueError):
                    pass
            try:
                rd, wr = idx["dram__bytes_read.sum"], idx["dram__bytes_write.sum"]
                dram_per_launch.append(float(r[rd]) * scale.get(units[rd], 1.0) + float(r[wr]) * scale.get(units[wr], 1.0))
            except (KeyError, ValueError):
                pass
    if a.launches:
        text = open(a.launches).read().splitlines()
        start = next(i for i, l in enumerate(text) if l.startswith('"ID"'))
        rows = list(csv.reader(io.StringIO("\n".join(text[start:]))))
        hdr = rows[0]
        ki, vi, gi, bi = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Grid Size"), hdr.index("Block Size")
        tot = defaultdict(float)
        cnt = defaultdict(int)
        for r in rows[1:]:
            name = r[ki].split("(")[0][:40]
            tot[name] += float(r[vi])
            cnt[name] += 1
        total = sum(tot.values())
        md += ["## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold, serialised)", "",
               "| kernel | launches | total ns | share |", "|---|---|---|---|"]
        for n in sorted(tot, key=lambda x: -tot[x]):
            md.append(f"| `{n}` | {cnt[n]} | {tot[n]:.0f} | {tot[n] / total:.3f} |")
        md.append("")
        md += ["First launches of the list:", "", "| id | kernel | grid | block | ns |", "|---|---|---|---|---|"]
        for r in rows[1:25]:
            md.append(f"| {r[0]} | `{r[ki].split('(')[0][:30]}` | {r[gi]} | {r[bi]} | {r[vi]} |")
        md.append("")
    with open(os.path.join(a.out, a.name + ".md"), "w") as fh:
        fh.write("\n".join(md) + "\n")
    sp = os.path.join(a.out, "ncu_summary.json")
    summ = json.load(open(sp)) if os.path.exists(sp) else {}
    if dram_per_launch:
        summ.setdefault(a.config, {})["dram_bytes_per_launch"] = sum(dram_per_launch) / len(dram_per_launch)
        summ[a.config]["source"] = a.name
    if alu_pct:
        summ.setdefault(a.config, {})["alu_pipe_pct"] = sum(alu_pct) / len(alu_pct)
    if dur_ns:
        summ.setdefault(a.config, {})["profiled_launch_ns"] = sum(dur_ns) / len(dur_ns)
    with open(sp, "w") as fh:
        json.dump(summ, fh, indent=1)


if __name__ == "__main__":
    main()
