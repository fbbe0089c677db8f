"""Static SASS opcode counts per kernel of libsynergy.so (offline evidence of the hardware paths:
tcgen05 MMA, TMEM loads, bulk copies, mbarriers, 256-bit block loads, L2 reductions).

    python scripts/sass_opcodes.py [OUT.md]      (default profiles/r2/s3_sass_opcodes.md)
"""
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sc_fandccfc23_b200", "libsynergy.so")
OPS = ["UTCIMMA", "UTCBAR", "LDTM", "UBLKCP", "UBLKPF", "UTMALDG", "SYNCS", "LDG.E.ENL2.256", "REDG.E.ADD.64",
       "ATOMS", "DFMA", "MUFU.RCP64H", "SHFL", "CREDUX"]


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r2", "s3_sass_opcodes.md")
    sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True, check=True).stdout
    lines = ["# SASS opcode evidence (`cuobjdump -sass` of libsynergy.so, sm_100a)", "",
             "Static instruction counts per kernel (a loop body counts once): `UTCIMMA` tcgen05 int8 MMA,",
             "`UTCBAR` tcgen05 commit, `LDTM` TMEM load, `UBLKCP` / `UBLKPF` bulk copy / L2 prefetch (TMA",
             "engine), `SYNCS` mbarrier, `LDG.E.ENL2.256` 32-byte block load, `REDG.E.ADD.64` L2 reduction,",
             "`CREDUX` warp min-reduction.  Regenerate: `python scripts/sass_opcodes.py`.", "",
             "| kernel | SASS instr. | " + " | ".join(f"`{o}`" for o in OPS) + " |",
             "|---|---|" + "---|" * len(OPS)]
    for f in sass.split("Function : ")[1:]:
        name = f.split("\n", 1)[0].strip()
        n = len(re.findall(r"^\s+/\*[0-9a-f]+\*/", f, re.M))
        cnt = [len(re.findall(r"\b" + re.escape(o), f)) for o in OPS]
        d = subprocess.run(["c++filt", name], capture_output=True, text=True).stdout.strip()
        d = re.sub(r"\(.*\)$", "", d.replace("syn::", "")).replace("void ", "")
        lines.append(f"| `{d}` | {n} | " + " | ".join(str(c) if c else "" for c in cnt) + " |")
    with open(out, "w") as fh:
        fh.write("\n".join(lines) + "\n")
    print(out)


if __name__ == "__main__":
    main()
