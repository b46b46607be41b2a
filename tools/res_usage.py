#!/usr/bin/env python3
"""Per-kernel registers / stack of libbsrng.so (cuobjdump -res-usage), demangled.

Usage: python tools/res_usage.py [path/to/libbsrng.so] [--max-stack N]
Exit status 1 if any kernel's stack exceeds --max-stack (default: report only).
"""
import re
import subprocess
import sys


def rows(lib):
    out = subprocess.run(["cuobjdump", "-res-usage", lib], capture_output=True, text=True).stdout
    names, res = [], []
    for ln in out.splitlines():
        m = re.search(r"Function (\S+):", ln)
        if m:
            names.append(m.group(1))
            continue
        m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+)", ln)
        if m and len(res) < len(names):
            res.append(tuple(int(x) for x in m.groups()))
    dem = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.splitlines()
    return [(d.replace("bsk::", "").replace("(KsArgs)", ""), *r) for d, r in zip(dem, res)]


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    lib = args[0] if args else "paper_conf_icppw_monfaredhkzrg20_b200/libbsrng.so"
    lim = None
    if "--max-stack" in sys.argv:
        lim = int(sys.argv[sys.argv.index("--max-stack") + 1])
    rs = sorted(rows(lib), key=lambda r: (-r[2], r[0]))
    print(f"{'REG':>4} {'STACK':>6} {'SMEM':>6}  kernel   ({len(rs)} kernels)")
    for name, reg, stack, smem in rs:
        print(f"{reg:4d} {stack:6d} {smem:6d}  {name}")
    if lim is not None and any(r[2] > lim for r in rs):
        sys.exit(1)


if __name__ == "__main__":
    main()
