"""Instruction mix of the hot loops of one kernel in libtbs.so (backward branches > 1 KB)."""
import re
import subprocess
import sys

lib = sys.argv[1]
pat = sys.argv[2]
txt = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
for f in re.split(r'\n\s+Function : ', txt):
    name = f.split('\n')[0]
    if pat not in name:
        continue
    print(name)
    lines = [l for l in f.split('\n') if re.search(r'/\*[0-9a-f]{4}\*/', l)]
    addr = lambda x: int(re.search(r'/\*([0-9a-f]{4,})\*/', x).group(1), 16)
    for l in lines:
        m = re.search(r'/\*([0-9a-f]{4,})\*/\s+(@!?U?P\w+\s+)?BRA(\.\S+)?\s+(?:!?U?P\w+,\s*)?(?:`?\(?)?0x([0-9a-f]+)', l)
        if m:
            src, dst = int(m.group(1), 16), int(m.group(4), 16)
            if dst < src and src - dst > 0x300:
                body = [x for x in lines if dst <= addr(x) <= src]
                ops = {}
                for x in body:
                    op = re.sub(r'/\*.*?\*/', '', x).strip().split()
                    o = op[0] if not op[0].startswith('@') else op[1]
                    o = o.split('.')[0]
                    ops[o] = ops.get(o, 0) + 1
                print(hex(dst), hex(src), len(body), sorted(ops.items(), key=lambda t: -t[1])[:14])
