"""Static SASS view of a kernel's hottest loop (the largest backward branch): opcode histogram,
issue slots vs ALU-pipe instructions, and the ALU/FMA/LDS pattern.  No GPU needed.

  python tools/sass_loop.py <file.o|.so> <mangled kernel name substring> [--pattern]
"""
import collections
import re
import subprocess
import sys

ALU = ("VABSDIFF4", "VIMNMX3", "VIMNMX", "IADD3", "LOP3", "SHF", "LEA", "ISETP", "VIADD", "SEL", "PRMT", "IMNMX",
       "FMNMX", "VIADDMNMX", "IABS", "FSEL", "PLOP3", "MOV")


def load(path, name):
    out = subprocess.run(["cuobjdump", "-sass", path], capture_output=True, text=True).stdout
    funcs = re.split(r"\n\s+Function : ", out)
    for f in funcs:
        head = f.split("\n", 1)[0]
        if name in head:
            return head.strip(), f
    raise SystemExit(f"{name} not found")


def main():
    path, name = sys.argv[1], sys.argv[2]
    head, body = load(path, name)
    ins = []
    for l in body.splitlines():
        m = re.match(r"\s+/\*([0-9a-f]{4,5})\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)([^;]*);", l)
        if m:
            ins.append((int(m.group(1), 16), m.group(3), m.group(4)))
    loops = []
    for a, op, args in ins:
        if op.startswith("BRA"):
            t = re.search(r"0x([0-9a-f]+)", args)
            if t and int(t.group(1), 16) < a:
                loops.append((int(t.group(1), 16), a))
    # the hottest loop = the innermost loop holding the most ALU work per instruction
    def density(lh):
        body = [op for a, op, _ in ins if lh[0] <= a <= lh[1]]
        n_alu = sum(1 for op in body if op.split(".")[0] in ALU and not op.startswith("IMAD"))
        return n_alu / max(1, len(body)), -len(body)
    lo, hi = max(loops, key=density)
    loop = [(a, op) for a, op, _ in ins if lo <= a <= hi]
    c = collections.Counter(op for _, op in loop)
    alu = sum(v for k, v in c.items() if k.split(".")[0] in ALU and not k.startswith("IMAD"))
    print(head)
    print(f"loop 0x{lo:x}..0x{hi:x}: {len(loop)} instructions, ALU-pipe {alu} ({2 * alu} ALU cycles/SMSP)")
    for k, v in c.most_common():
        print(f"  {v:5d} {k}")
    if "--pattern" in sys.argv:
        key = {"VABSDIFF4": "A", "VIMNMX3": "M", "IMAD": "I", "LDS": "L"}
        s = "".join(key.get(op.split(".")[0], "o") for _, op in loop)
        for i in range(0, len(s), 100):
            print(s[i:i + 100])


if __name__ == "__main__":
    main()
