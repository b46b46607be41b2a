#!/usr/bin/env python3
"""Render tools/sweep_c5.py JSONL output as the markdown tables in
profiles/<round>_sweep_c5.md.   Usage: sweep_summary.py sweep.jsonl [curand.log]"""
import json
import sys
from collections import defaultdict


def fmt_n(n):
    return f"2^{n.bit_length() - 1}" if n & (n - 1) == 0 else str(n)


def main():
    rows = [json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
    out = []
    sched = [r for r in rows if r.get("sweep") == "schedule"]
    if sched:
        out.append("### Schedule x occupancy x instances x clocks per launch (MICKEY 2.0, consume)\n")
        out.append("Tb/s (fraction of the ALU roofline at the sampled SM clock). `paper_oneshot` = one thread per "
                   "32-instance group for the whole call (the paper's launch style); `persist_1w`/`persist_2w` = "
                   "persistent time-segmented queue with 1 / 2 clock-loop warps per SMSP; `auto` = the library "
                   "default.\n")
        names = ["paper_oneshot", "persist_1w", "persist_2w", "auto"]
        out.append("| n | clocks/launch | " + " | ".join(names) + " |")
        out.append("|---|---|" + "---|" * len(names))
        grid = defaultdict(dict)
        for r in sched:
            grid[(r["n"], r["clocks_per_call"])][r["schedule"]] = r
        for (n, c), d in sorted(grid.items()):
            cells = [f"{d[k]['tbps']:.3f} ({d[k]['alu_frac']:.3f})" if k in d else "-" for k in names]
            out.append(f"| {fmt_n(n)} | {c} | " + " | ".join(cells) + " |")
        out.append("")
    for sw, title in (("unroll", "Clocks unrolled per loop iteration U (MICKEY 2.0, n = 2^22, 2^16 clocks)"),
                      ("layout", "Output layouts (MICKEY 2.0, n = 2^22, 2^16 clocks)"),
                      ("rm_staging", "ROW_MAJOR staging variants (n = 2^22, 2^15-bit calls = 4 KB rows)"),
                      ("cipher", "Grain v1 / AES-128-CTR occupancy and unroll (n = 2^22, 2^16 clocks)")):
        sel = [r for r in rows if r.get("sweep") == sw]
        if not sel:
            continue
        out.append(f"### {title}\n")
        out.append("| cipher | layout | clocks/call | options | ms | Tb/s | ALU frac (kernel ops) | ALU frac (sec. 8(d) ops) | HBM writes GB/s | SM MHz |")
        out.append("|---|---|---|---|---|---|---|---|---|---|")
        for r in sel:
            opts = (r.get("staging", "") + ": " if r.get("staging") else "") + \
                (", ".join(f"{k}={v}" for k, v in r["opts"].items()) or "default")
            alg = r.get("alu_frac_alg")
            hbm = r.get("hbm_write_gbs")
            out.append(f"| {r['cipher']} | {r['layout']} | {r['clocks_per_call']} | {opts} | {r['ms']} | "
                       f"{r['tbps']:.3f} | {r['alu_frac']:.3f} | {alg if alg is not None else '-'} | "
                       f"{hbm if hbm is not None else '-'} | {r['sm_mhz']} |")
        out.append("")
    if len(sys.argv) > 2:
        out.append("### cuRAND on the same B200 (context)\n")
        out.append("| generator | API | bytes / bits | ms | Tb/s | HBM write GB/s |")
        out.append("|---|---|---|---|---|---|")
        for l in open(sys.argv[2]):
            if not l.startswith("{"):
                continue
            d = json.loads(l)
            size = d.get("bytes", d.get("bits"))
            out.append(f"| {d['curand']} | {d['api']} | {size} | {d['ms']} | {d['tbps']:.2f} | "
                       f"{d.get('hbm_write_gbs', '-')} |")
        out.append("")
    print("\n".join(out))


if __name__ == "__main__":
    main()
