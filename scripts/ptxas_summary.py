"""Per-kernel registers / spills from `nvcc -Xptxas -v` output (stdin)."""
import re
import subprocess
import sys

text = sys.stdin.read()
cur = None
rows = []
for line in text.splitlines():
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur = m.group(1)
        continue
    m = re.search(r"(\d+) bytes spill stores", line)
    if m and cur:
        spill = int(m.group(1))
    m2 = re.search(r"Used (\d+) registers", line)
    if m2 and cur:
        name = subprocess.run(["c++filt", cur], capture_output=True, text=True).stdout.strip()
        name = re.sub(r"mega::kern::|\(mega::kern::\w+\)", "", name).replace("void ", "")
        rows.append((name, int(m2.group(1)), spill))
        cur = None
pat = sys.argv[1] if len(sys.argv) > 1 else ""
for n, r, s in rows:
    if re.search(pat, n):
        print(f"{r:4d} regs  spill {s:5d}  {n}")
