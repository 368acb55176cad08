"""Static SASS instructions per CUDA source line of one kernel in libgsnp.so (I-cache budget).
usage: python tools/static_lines.py [mangled-name-substring] [topN]"""
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
name = sys.argv[1] if len(sys.argv) > 1 else "_ZN8gsnp_dev11k_call_tileILb0ELi32E"
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
lib = os.path.abspath(os.environ.get("GSNP_LIB") or "") if os.environ.get("GSNP_LIB") else os.path.join(ROOT, "paper_conf_icpp_luzlwfl11_b200", "libgsnp.so")
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=d, capture_output=True)
txt = ""
for f in os.listdir(d):
    if f.endswith(".cubin"):
        txt += subprocess.run(["nvdisasm", "-g", os.path.join(d, f)], capture_output=True, text=True).stdout
i = txt.index(".text." + [m for m in re.findall(r"\.text\.(\S+):", txt) if name in m][0] + ":")
j = txt.find(".text.", i + 10)
cur, cnt, n = None, {}, 0
for line in txt[i:j].splitlines():
    m = re.search(r'//## File ".*?/([^/"]+)", line (\d+)', line)
    if m:
        cur = (m.group(1), int(m.group(2)))
        continue
    if re.match(r"\s+/\*[0-9a-f]{4,}\*/", line):
        cnt[cur] = cnt.get(cur, 0) + 1
        n += 1
print("static instructions", n)
for k, v in sorted(cnt.items(), key=lambda x: -x[1])[:top]:
    print(f"{v:6d}  {k}")
