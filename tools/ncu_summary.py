#!/usr/bin/env python3
"""Summarise a gpurun_out/prof capture (tools/gpu_profile.sh) into profiles/.

  python tools/ncu_summary.py gpurun_out/prof r1
writes profiles/<tag>_launches.csv, <tag>_launch_shares.md, <tag>_<rep>_metrics.csv,
<tag>_summary.md and keystream_traffic.json (read by bench.py)."""
import csv
import io
import json
import os
import shutil
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "launch__grid_size", "launch__block_size",
    "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.per_cycle_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_alu.sum", "smsp__inst_executed.sum", "smsp__issue_active.avg.per_cycle_active",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_op_write.sum", "smsp__sass_inst_executed_op_local_ld.sum",
    "smsp__sass_inst_executed_op_local_st.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
              "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1, "second": 1}


def raw_metrics(rep):
    if rep.endswith(".csv"):
        txt = open(rep).read()
    else:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    out = []
    for row in rows[2:]:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        out.append({k: (d[k], u.get(k, "")) for k in hdr})
    return out


def num(v):
    return float(str(v).replace(",", ""))


def si(val_unit):
    v, u = val_unit
    return num(v) * UNIT_SCALE.get(u, 1)


def main():
    src, tag = sys.argv[1], sys.argv[2]
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    lines = [f"# {tag} ncu summary\n", f"Source: `{src}` (tools/gpu_profile.sh); GPU: "
             + open(os.path.join(src, "gpu.txt")).read().strip().replace("\n", " / ") + "\n"]

    # launch list
    lc = os.path.join(src, "launches.csv")
    if os.path.exists(lc):
        shutil.copy(lc, os.path.join(prof, f"{tag}_launches.csv"))
        rows = list(csv.reader(open(lc)))
        i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
        hdr = rows[i]
        agg = defaultdict(lambda: [0, 0.0])
        for r in rows[i + 1:]:
            d = dict(zip(hdr, r))
            if d.get("Metric Name") != "gpu__time_duration.sum":
                continue
            k = d["Kernel Name"].split("(")[0]
            agg[k][0] += 1
            agg[k][1] += num(d["Metric Value"]) * UNIT_SCALE.get(d["Metric Unit"], 1e-9)
        tot = sum(v[1] for v in agg.values())
        lines.append("\n## Launch list of `python bench.py --no-cpu-baseline --no-context` "
                     "(ncu gpu__time_duration, cold-cache, serialised)\n")
        lines.append("| kernel | launches | total s | share |\n|---|---|---|---|")
        for k, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
            lines.append(f"| `{k}` | {c} | {v:.4f} | {100 * v / tot:.2f}% |")
        with open(os.path.join(prof, f"{tag}_launch_shares.md"), "w") as f:
            f.write("\n".join(lines[2:]) + "\n")

    traffic = {}
    for rep in sorted(os.listdir(src)):
        if rep.endswith(".ncu-rep"):
            name = rep[:-8]
        elif rep.endswith("_raw.csv"):
            name = rep[:-8]
        else:
            continue
        ms = raw_metrics(os.path.join(src, rep))
        if not ms:
            continue
        m = ms[0]
        with open(os.path.join(prof, f"{tag}_{name}_metrics.csv"), "w", newline="") as f:
            w = csv.writer(f)
            w.writerow(["metric", "value", "unit"])
            for k in KEYS:
                if k in m:
                    w.writerow([k, m[k][0], m[k][1]])
        logf = [os.path.join(src, f"ncu_{name}.log"), os.path.join(src, f"ncu_{name.replace('ks_', '')}.log")]
        logf = [f for f in logf if os.path.exists(f)]
        log = open(logf[0]).read() if logf else ""
        lines.append(f"\n## `{name}` — {m.get('Kernel Name', ('?', ''))[0][:100]}\n")
        argline = [ln for ln in log.splitlines() if ln.startswith("done Namespace")]
        if argline:
            lines.append(f"driver: `{argline[-1]}`\n")
        lines.append("| metric | value | unit |\n|---|---|---|")
        for k in KEYS:
            if k in m:
                lines.append(f"| {k} | {m[k][0]} | {m[k][1]} |")
        rd, wr = si(m["dram__bytes_read.sum"]), si(m["dram__bytes_write.sum"])
        traffic[name] = {"dram_read": rd, "dram_write": wr, "duration_s": si(m["gpu__time_duration.sum"]),
                         "driver": argline[-1] if argline else None}
    with open(os.path.join(prof, f"{tag}_summary.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    if "ks_consume" in traffic:
        t = traffic["ks_consume"]
        t = dict(t)
        json.dump({"mode": "consume", "n": 1 << 22,
                   "dram_bytes_per_launch": t["dram_read"] + t["dram_write"],
                   "note": ("ncu --set full capture of keystream_kernel<CHECKSUM> at n=2^22, 2^16 bits "
                            f"({tag}); at the bench's 2^20 bits the launch has the same work items (one per "
                            "warp-unit, state carry 100 MiB in + 100 MiB out), so bytes per launch match"),
                   "captures": traffic}, open(os.path.join(prof, "keystream_traffic.json"), "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
