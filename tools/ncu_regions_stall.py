"""Stall-reason breakdown per kernel region (source-line ranges) of one
ncu --set full report:  python tools/ncu_regions_stall.py REP LIB KERNEL_SUBSTR REGIONS.json
REGIONS.json = [["name", first_line, last_line], ...] (lines of the kernel's own file;
inlined helpers are charged to their call site)."""
import collections, csv, json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(__file__))
os.environ["NCU_LINES_CALLSITE"] = "1"
import ncu_lines

rep, lib, kern, regf = sys.argv[1:5]
regs = json.load(open(regf))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
rows = [r for r in rows[2:] if len(r) > 5 and r[0].startswith("0x")]
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
ie = hdr.index("Instructions Executed")
base = int(rows[0][0], 16)
tab = ncu_lines.line_table(lib, kern)
acc = collections.defaultdict(lambda: collections.Counter())
for r in rows:
    off = int(r[0], 16) - base
    src = tab.get(off, (("?", 0), ""))[0]
    name = "other"
    for nm, a, b in regs:
        if a <= src[1] <= b and src[0].endswith(".cuh"):
            name = nm
            break
    c = acc[name]
    c["instr"] += int(r[ie] or 0)
    for i in stall_cols:
        c[hdr[i]] += int(r[i] or 0)
tot = sum(sum(v for k, v in c.items() if k != "instr") for c in acc.values())
for name, c in sorted(acc.items(), key=lambda kv: -sum(v for k, v in kv[1].items() if k != "instr")):
    s = sum(v for k, v in c.items() if k != "instr")
    top = ", ".join(f"{k[6:]} {100*v/max(s,1):.0f}%" for k, v in c.most_common(8) if k != "instr")
    print(f"{name:10s} samples {100*s/tot:5.1f}%  instr {c['instr']/1e9:6.2f}e9  | {top}")
