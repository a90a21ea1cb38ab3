"""Register / spill table of the hot kernel instantiations from a ptxas -v log.

    python tools/regs.py [paper_conf_ipps_fanwc23_b200/ptxas.log]
"""
import re
import subprocess
import sys


def table(path):
    txt = open(path).read().splitlines()
    out, cur = [], None
    for line in txt:
        m = re.search(r"Compiling entry function '(\S+)'", line)
        if m:
            cur = m.group(1)
            spill = None
            continue
        m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
        if m and cur:
            spill = int(m.group(1)) + int(m.group(2))
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            out.append((cur, int(m.group(1)), spill))
            cur = None
    return out


def demangle(names):
    r = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True)
    return r.stdout.splitlines()


if __name__ == "__main__":
    rows = table(sys.argv[1] if len(sys.argv) > 1 else
                 "paper_conf_ipps_fanwc23_b200/ptxas.log")
    names = demangle([r[0] for r in rows])
    for (m, regs, sp), n in zip(rows, names):
        if "spmm_kernel" in n or "sddmm_kernel" in n:
            n = re.sub(r"\(.*", "", n).replace("gnn::", "")
            print(f"{regs:4d} regs  spill {sp or 0:5d} B  {n}")
