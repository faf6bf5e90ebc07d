#!/usr/bin/env python
"""Summarise an `ncu --set full` report (one bench step) into profiles/<round>/:
a markdown table of the key counters per kernel and latest_gather_ncu.json (the
gather kernel's DRAM traffic per launch, read by bench.py's roofline.traffic).

    python profiles/summarize_ncu.py gpurun_out/prof_step.ncu-rep profiles/r02 [rows_gathered] [workload]
"""

import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "time_us"),
    ("dram__bytes_read.sum", "dram_read_MB"),
    ("dram__bytes_write.sum", "dram_write_MB"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct"),
    ("lts__t_sector_hit_rate.pct", "l2_hit_pct"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_pct"),
    ("launch__grid_size", "grid"),
    ("launch__registers_per_thread", "regs"),
    ("launch__occupancy_limit_registers", "occ_limit_regs"),
    ("lts__t_requests_op_atom_dot_cas.sum", "l2_cas_requests"),
    ("lts__t_sectors_op_atom.sum", "l2_atom_sectors"),
]


def sectors_per_request(r, idx):
    """global-load sectors per request (4 = a fully used 128 B line per warp request of 32 x 4 B)."""
    s, q = "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum"
    try:
        return f"{float(r[idx[s]].replace(',', '')) / float(r[idx[q]].replace(',', '')):.2f}"
    except (KeyError, ValueError, ZeroDivisionError):
        return ""


def main():
    rep, outdir = sys.argv[1], sys.argv[2]
    rows_gathered = float(sys.argv[3]) if len(sys.argv) > 3 else None
    workload = sys.argv[4] if len(sys.argv) > 4 else "products"
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    idx = {k: j for j, k in enumerate(hdr)}
    stall = [k for k in hdr if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio")]
    os.makedirs(outdir, exist_ok=True)
    md = ["| # | kernel | " + " | ".join(n for _, n in KEYS) + " | ld_sectors_per_request | top stalls (cycles/issue) |",
          "|---|---|" + "---|" * len(KEYS) + "---|---|"]
    gather = None
    for n, r in enumerate(data):
        name = r[idx["Kernel Name"]]
        vals = []
        for k, _ in KEYS:
            vals.append(r[idx[k]] if k in idx else "")
        st = sorted(((float(r[idx[k]] or 0), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")])
                     for k in stall), reverse=True)[:3]
        md.append(f"| {n} | `{name[:48]}` | " + " | ".join(vals) + f" | {sectors_per_request(r, idx)} | " +
                  ", ".join(f"{s}={v:.1f}" for v, s in st) + " |")
        if "gather_kernel" in name or "gather_dense_kernel" in name:
            rd = float(r[idx["dram__bytes_read.sum"]])
            wr = float(r[idx["dram__bytes_write.sum"]])
            unit = units[idx["dram__bytes_read.sum"]]
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1e6)
            gather = {"kernel": name, "dram_read_bytes": rd * scale, "dram_write_bytes": wr * scale,
                      "dram_bytes_per_launch": (rd + wr) * scale,
                      "time_us": float(r[idx["gpu__time_duration.sum"]]), "report": os.path.basename(rep)}
            if rows_gathered:
                gather["rows_gathered"] = rows_gathered
    with open(os.path.join(outdir, "ncu_step_summary.md"), "w") as f:
        f.write(f"ncu --set full, one bench step (report {os.path.basename(rep)}; units: us, MB, %)\n\n")
        f.write("\n".join(md) + "\n")
    if gather:
        with open(os.path.join(outdir, "gather_ncu.json"), "w") as f:
            json.dump(gather, f, indent=1)
        latest = os.path.join(os.path.dirname(outdir.rstrip("/")), "latest_gather_ncu.json")
        try:
            with open(latest) as f:
                allw = json.load(f)
            allw = allw if "kernel" not in allw else {}
        except (OSError, ValueError):
            allw = {}
        allw[workload] = gather
        with open(latest, "w") as f:
            json.dump(allw, f, indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
