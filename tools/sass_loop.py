"""Instruction histogram of an address range of a cuobjdump -sass listing (loop inspection).
usage: python tools/sass_loop.py file.sass FUNC_SUBSTR START_HEX END_HEX [SKIP_START SKIP_END ...]"""
import re
import sys
from collections import Counter

path, func, a, b = sys.argv[1], sys.argv[2], int(sys.argv[3], 16), int(sys.argv[4], 16)
skips = [(int(sys.argv[i], 16), int(sys.argv[i + 1], 16)) for i in range(5, len(sys.argv), 2)]
inside = False
c = Counter()
n = 0
for line in open(path):
    if "Function :" in line:
        inside = func in line
        continue
    if not inside:
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if not m:
        continue
    addr = int(m.group(1), 16)
    if not (a <= addr < b) or any(s <= addr < e for s, e in skips):
        continue
    ins = m.group(2).split()
    op = ins[1] if ins[0].startswith("@") else ins[0]
    c[op] += 1
    n += 1
for op, k in c.most_common():
    print(f"{k:5d} {op}")
print(f"{n:5d} TOTAL")
