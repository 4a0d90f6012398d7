"""Per-function SASS statistics of a cubin/.so: python tools/sass_stats.py LIB [name-substring]"""
import re
import subprocess
import sys

txt = subprocess.run(["cuobjdump", "-sass", sys.argv[1]], capture_output=True, text=True).stdout
pat = sys.argv[2] if len(sys.argv) > 2 else ""
blocks = re.split(r"\n\s*Function : ", txt)
for b in blocks[1:]:
    name = b.split("\n", 1)[0].strip()
    if pat not in name:
        continue
    ins = re.findall(r"/\*[0-9a-f]{4,}\*/\s+([^;]*);", b)
    ops = [i.split()[0] if not i.startswith("@") else i.split()[1] for i in ins if i.strip()]
    from collections import Counter
    c = Counter(o.split(".")[0] for o in ops)
    keys = ["LDG", "STG", "LDS", "STS", "LDL", "STL", "SYNCS", "BAR", "SHFL", "UBLKCP", "UTMALDG", "CALL", "RET", "MEMBAR", "ATOMG", "RED"]
    print(name[:100], "n=%d" % len(ops), " ".join(f"{k}={c.get(k, 0)}" for k in keys))
