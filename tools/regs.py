"""Registers / spills / smem per kernel from the nvcc -Xptxas -v logs."""
import re, subprocess, sys, glob
for log in sorted(glob.glob('build/obj/*.log')):
    txt = open(log).read()
    for m in re.finditer(r"Compiling entry function '(\S+)' for 'sm_100a'\n(.*?)(?=Compiling entry|\Z)", txt, re.S):
        body = m.group(2)
        regs = re.search(r"Used (\d+) registers", body)
        spill = re.search(r"(\d+) bytes spill stores", body)
        smem = re.search(r"(\d+) bytes smem", body)
        name = subprocess.run(['c++filt', m.group(1)], capture_output=True, text=True).stdout.strip()
        name = name.replace('sfs::(anonymous namespace)::', '').split('(')[0]
        if len(sys.argv) > 1 and sys.argv[1] not in name:
            continue
        print(f"{regs.group(1) if regs else '?':>4} regs {spill.group(1) if spill else '0':>4} spill {smem.group(1) if smem else '0':>6} smem  {name}")
