"""Per-region instruction / sample shares of one kernel from an ncu report.

  python tools/ncu_regions.py REPORT LIB KERNEL_SUBSTR name:lo:hi ...
Regions are line ranges of the kernel's main .cuh file (inlined helpers keep
their own lines and are listed separately by file)."""
import subprocess
import sys
import re

rep, lib, kern = sys.argv[1:4]
out = subprocess.run([sys.executable, "tools/ncu_lines.py", rep, lib, kern, "100000"], capture_output=True,
                     text=True).stdout
rng = [(a.split(":")[0], int(a.split(":")[1]), int(a.split(":")[2])) for a in sys.argv[4:]]
main = None
agg, fagg = {}, {}
tot = None
for l in out.splitlines():
    if l.startswith("samples"):
        tot = l
        continue
    m = re.match(r"(\S+?)(\(wait\))?:(\d+)\s+([\d.]+)\s+([\d.]+)", l)
    if not m:
        continue
    f, w, ln, s, i = m.group(1), m.group(2), int(m.group(3)), float(m.group(4)), float(m.group(5))
    key = None
    if f == "monitor_fused.cuh":
        for name, a, b in rng:
            if a <= ln <= b:
                key = name
    if key is None:
        key = f + ("(wait)" if w else "")
    v = agg.setdefault(key, [0.0, 0.0])
    v[0] += s
    v[1] += i
print(tot)
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k:28s} samples {v[0]:6.2f}%  instr {v[1]:6.2f}%")
