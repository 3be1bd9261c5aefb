"""Opcode histogram of one kernel's SASS in libmimose.so (static counts):
python tools/sass_hist.py <function-name-substring>"""
import collections
import re
import subprocess
import sys

so = "paper_conf_ipps_liaolysshfyctzlq23_b200/libmimose.so"
out = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
fn, cnt = None, collections.Counter()
for ln in out.splitlines():
    m = re.search(r"Function : (\S+)", ln)
    if m:
        if fn:
            break
        fn = m.group(1) if sys.argv[1] in m.group(1) else None
        continue
    if fn:
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", ln)
        if m:
            cnt[m.group(2)] += 1
print(fn, sum(cnt.values()))
for op, c in cnt.most_common(30):
    print(f"{op:12s} {c}")
