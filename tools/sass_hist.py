"""Opcode histogram of a kernel's loops from its SASS (no GPU needed).

    python tools/sass_hist.py <file.cu> <kernel-substring> [min_loop_len] [nvcc flags...]

Compiles the .cu to a cubin for sm_100a (same flags as the product build),
finds every backward branch in the kernel, and prints each loop body of at
least min_loop_len instructions with its opcode counts and per-pipe split
(ALU: LOP3/SHF/LEA/PRMT/IADD3/ISETP/SEL...; FMA-heavy: IMAD*/VIADD, measured
with tools/microbench_pipes.cu)."""
import collections
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ALU = ("LOP3", "SHF", "LEA", "PRMT", "IADD3", "ISETP", "SEL", "FLO", "POPC", "BMSK", "PLOP3",
       "IABS", "IMNMX", "VIMNMX", "BREV", "SGXT", "LOP")
FMA = ("IMAD", "VIADD", "IMUL")


def pipe(op):
    base = op.split(".")[0]
    if base in ALU:
        return "alu"
    if base in FMA:
        return "fma"
    if base in ("LDS", "STS", "LDG", "STG", "LD", "ST", "ATOMS", "ATOMG", "RED", "SHFL", "LDSM"):
        return "lsu"
    return "other"


def main():
    src, kname = sys.argv[1], sys.argv[2]
    min_len = int(sys.argv[3]) if len(sys.argv) > 3 else 100
    extra = sys.argv[4:]
    with tempfile.TemporaryDirectory() as td:
        cub = os.path.join(td, "k.cubin")
        subprocess.check_call(["nvcc", "-O3", "-std=c++17", "-lineinfo", "-gencode",
                               "arch=compute_100a,code=sm_100a", "-cubin", "-I",
                               os.path.join(ROOT, "include"), "-o", cub, *extra, src])
        sass = subprocess.check_output(["cuobjdump", "-sass", cub], text=True)
    for m in re.finditer(r"Function : (\S+)", sass):
        if not re.search(kname, m.group(1)):
            continue
        i = m.end()
        j = sass.find("Function :", i)
        body = sass[i:j if j > 0 else None]
        ins = [(int(a, 16), s) for a, s in
               re.findall(r"/\*([0-9a-f]{4,5})\*/\s+((?:@!?U?P\w+\s+)?[A-Z0-9_.]+[^;]*);", body)]
        print(f"== {m.group(1)}: {len(ins)} instructions")
        for a, s in ins:
            b = re.search(r"BRA(?:\.U)?\s+(?:!?U?P\w+,\s*)?0x([0-9a-f]+)", s)
            if not b or int(b.group(1), 16) >= a:
                continue
            t = int(b.group(1), 16)
            loop = [x for y, x in ins if t <= y <= a]
            if len(loop) < min_len:
                continue
            c = collections.Counter()
            pc = collections.Counter()
            for x in loop:
                w = x.split()
                op = w[1] if w[0].startswith("@") else w[0]
                c[op] += 1
                pc[pipe(op)] += 1
            print(f"  loop {t:#x}..{a:#x}: {len(loop)} instr, pipes {dict(pc)}")
            print("   ", ", ".join(f"{k} {v}" for k, v in c.most_common(14)))


if __name__ == "__main__":
    main()
