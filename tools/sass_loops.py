#!/usr/bin/env python3
"""SASS audit: per kernel, find backward branches (loops) and histogram the
opcodes of each loop body.  Usage: sass_loops.py <cubin|so> [kernel-substring]"""
import re
import subprocess
import sys
from collections import Counter

def main():
    path = sys.argv[1]
    filt = sys.argv[2] if len(sys.argv) > 2 else ""
    txt = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True, check=True).stdout
    funcs = re.split(r"\n\s+Function : ", txt)[1:]
    for f in funcs:
        name = f.split("\n", 1)[0].strip()
        if filt not in name:
            continue
        ins = []
        for m in re.finditer(r"/\*([0-9a-f]{4,})\*/\s+([^;]*);", f):
            ins.append((int(m.group(1), 16), m.group(2).strip()))
        print(f"== {name}: {len(ins)} instructions")
        total = Counter(re.sub(r"^@!?U?P\w+\s+", "", t).split()[0].split(".")[0] for _, t in ins)
        print("   whole kernel:", dict(total.most_common(12)))
        for addr, t in ins:
            m = re.search(r"BRA(?:\.\w+)*\s+(?:!?U?P\w+,\s*)?(0x[0-9a-f]+)", t)
            if not m:
                continue
            tgt = int(m.group(1), 16)
            if tgt >= addr:
                continue
            body = [x for a, x in ins if tgt <= a <= addr]
            c = Counter(re.sub(r"^@!?U?P\w+\s+", "", x).split()[0].split(".")[0] for x in body)
            print(f"   loop 0x{tgt:x}-0x{addr:x} ({len(body)} instr):", dict(c.most_common(12)))

if __name__ == "__main__":
    main()
