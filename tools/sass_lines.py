"""Static SASS size of one kernel by source line: python tools/sass_lines.py file.cubin KERNEL_SUBSTR [N]
(nvdisasm --print-line-info; counts instructions attributed to each file:line)."""
import re
import subprocess
import sys
from collections import Counter

cub, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["nvdisasm", "--print-line-info", "-c", cub], capture_output=True, text=True).stdout
cur_fn, line, cnt, total = None, None, Counter(), 0
for l in out.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", l)
    if m:
        cur_fn = m.group(1)
        continue
    if cur_fn is None or kern not in cur_fn:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        line = f"{m.group(1).split('/')[-1]}:{m.group(2)}"
        continue
    if re.match(r"\s*/\*[0-9a-f]{4,}\*/", l):
        cnt[line] += 1
        total += 1
print("total", total)
for k, v in cnt.most_common(top):
    print(f"{v:6d} {k}")
