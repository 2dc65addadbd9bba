"""Instruction mix of a sweep kernel's column steps from its SASS (cuobjdump -sass -fun NAME lib.so).

Splits the listing at VOTE.ANY (one per column step) and prints, for the step
blocks that hold the FMNMX3 column minimum, the length and opcode histogram.
    python tools/sass_steps.py FILE.sass
"""
import collections
import re
import sys

ins = []
for line in open(sys.argv[1]):
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        s = m.group(2).strip()
        op = s.split()[1] if s.startswith("@") else s.split()[0]
        ins.append(op.split(".")[0])
votes = [k for k, op in enumerate(ins) if op == "VOTE"]
for a, b in zip(votes, votes[1:]):
    seg = ins[a + 1:b + 1]
    if "FMNMX3" in seg and "FFMA2" in seg and len(seg) < 160:
        h = collections.Counter(seg)
        print(len(seg), dict(sorted(h.items(), key=lambda kv: -kv[1])))
