#!/usr/bin/env python
"""Summarise ncu reports (--set full captures) into a markdown table and a
traffic.json (DRAM bytes per launch per kernel), for profiles/.

    python tools/ncu_summarize.py OUT_DIR name=path.ncu-rep [...]
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    "sm__inst_executed.sum": "inst_executed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
    "launch__registers_per_thread": "regs",
    "launch__shared_mem_per_block_dynamic": "dyn_smem",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "lts__t_bytes.sum": "l2_bytes",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum": "smem_bank_conflicts",
    "smsp__inst_executed_pipe_fma.sum": "pipe_fma_inst",
    "smsp__inst_executed_pipe_alu.sum": "pipe_alu_inst",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active": "alu_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "fma_pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum": "smem_wavefronts",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed": "smem_pct",
    "lts__t_sectors.sum": "l2_sectors",
}
SCALE = {"Kbyte/block": 1e3, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1, "Tbyte": 1e12,
         "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}


def read(rep):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k, name in KEYS.items():
            if k in hdr:
                i = hdr.index(k)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                d[name] = v * SCALE.get(units[i], 1)
        out.append(d)
    return out


def main():
    outdir = sys.argv[1]
    os.makedirs(outdir, exist_ok=True)
    if len(sys.argv) > 2 and sys.argv[2].startswith("--compare="):
        return compare(outdir, sys.argv[2].split("=", 1)[1], sys.argv[3:])
    table = ["| capture | kernel | duration (us) | DRAM read (MB) | DRAM write (MB) | DRAM % peak | SM % | "
             "issue active % | warps active % | regs | grid x block | smem/CTA (KB) |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    traffic = {}
    for arg in sys.argv[2:]:
        name, rep = arg.split("=", 1)
        for d in read(rep):
            k = d["kernel"].split("(")[0].split("<")[0].replace("void ", "").strip()
            table.append(
                f"| {name} | `{k}` | {d.get('duration', 0) * 1e6:.1f} | {d.get('dram_read', 0) / 1e6:.1f} | "
                f"{d.get('dram_write', 0) / 1e6:.1f} | {d.get('dram_pct', 0):.1f} | {d.get('sm_pct', 0):.1f} | "
                f"{d.get('issue_active_pct', 0):.1f} | {d.get('occupancy_pct', 0):.1f} | {d.get('regs', 0):.0f} | "
                f"{d.get('grid', 0):.0f} x {d.get('block', 0):.0f} | {d.get('dyn_smem', 0) / 1e3:.1f} |")
            traffic[name] = {"kernel": k, "dram_bytes_per_launch": d.get("dram_read", 0) + d.get("dram_write", 0),
                             "dram_read": d.get("dram_read", 0), "dram_write": d.get("dram_write", 0),
                             "duration_s_under_ncu": d.get("duration", 0), "source": os.path.basename(rep)}
    with open(os.path.join(outdir, "ncu_summary.md"), "w") as f:
        f.write("\n".join(table) + "\n")
    with open(os.path.join(outdir, "traffic.json"), "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(table))


def compare(outdir, fname, args):
    """Variant comparison table (pipe/issue/memory utilisation side by side)."""
    table = ["| capture | kernel | duration (us) | issue active % | ALU pipe % | FMA pipe % | smem wavefronts % | "
             "DRAM read (MB) | DRAM % peak | L2 bytes (MB) | warps active % | regs |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for arg in args:
        name, rep = arg.split("=", 1)
        if not os.path.exists(rep):
            table.append(f"| {name} | (no capture) |" + " |" * 10)
            continue
        for d in read(rep):
            k = d["kernel"].split("(")[0].split("<")[0].replace("void ", "").strip()
            table.append(
                f"| {name} | `{k}` | {d.get('duration', 0) * 1e6:.1f} | {d.get('issue_active_pct', 0):.1f} | "
                f"{d.get('alu_pct', 0):.1f} | {d.get('fma_pct', 0):.1f} | {d.get('smem_pct', 0):.1f} | "
                f"{d.get('dram_read', 0) / 1e6:.1f} | {d.get('dram_pct', 0):.1f} | {d.get('l2_sectors', 0) * 32 / 1e6:.1f} | "
                f"{d.get('occupancy_pct', 0):.1f} | {d.get('regs', 0):.0f} |")
    with open(os.path.join(outdir, fname), "w") as f:
        f.write("\n".join(table) + "\n")
    print("\n".join(table))


if __name__ == "__main__":
    main()
