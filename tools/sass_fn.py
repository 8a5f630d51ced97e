"""Per-function SASS statistics of the fused kernel (device functions live in
the kernel's section; symbols give their offset/size).

    python tools/sass_fn.py paper_conf_sc_panzzxwslr0d24_b200/build_obj/fused_k4.cu.o sched_groupILi3E [--dump]
"""
import re
import subprocess
import sys
from collections import Counter


def main():
    obj, pat = sys.argv[1], sys.argv[2]
    dump = '--dump' in sys.argv
    elf = subprocess.run(['cuobjdump', '-elf', obj], capture_output=True, text=True).stdout
    syms = []
    for line in elf.splitlines():
        m = re.match(r'\s*0x[0-9a-f]+\s+0x([0-9a-f]+)\s+0x([0-9a-f]+)\s+0x2\s+\S+\s+\S+\s+\$\S+\$(\S+)', line)
        if m:
            syms.append((int(m.group(1), 16), int(m.group(2), 16), m.group(3)))
    sass = subprocess.run(['cuobjdump', '-sass', obj], capture_output=True, text=True).stdout
    ins = []
    for line in sass.splitlines():
        m = re.match(r'\s+/\*([0-9a-f]{4,})\*/\s+(.*?);', line)
        if m:
            ins.append((int(m.group(1), 16), m.group(2).strip()))
    for off, size, name in syms:
        if pat not in name:
            continue
        body = [t for a, t in ins if off <= a < off + size]
        ops = Counter(re.sub(r'^@!?U?P\w+\s+', '', t).split()[0].split('.')[0] for t in body)
        print(f'{name[:90]}  n={len(body)}  LDL={ops["LDL"]} STL={ops["STL"]} LDG={ops["LDG"]} '
              f'FADD={ops["FADD"]} FFMA={ops["FFMA"]} PRMT={ops["PRMT"]} SHFL={ops["SHFL"]}')
        if dump:
            for t in body:
                print('   ', t)


if __name__ == '__main__':
    main()
