"""Per-source-line profile of one kernel: joins ncu's per-SASS-instruction
samples / executed counts (source page) with the cubin's line table
(nvdisasm -g), since ncu's own CUDA view loses inlined helper lines.

  python tools/ncu_lines.py REPORT.ncu-rep LIB.so KERNEL_SUBSTR [top]
"""
import collections
import csv
import os
import re
import subprocess
import sys
import tempfile


def sass_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = [r for r in csv.reader(out.splitlines())][2:]
    return [r for r in rows if len(r) > 5 and r[0].startswith("0x")]


def line_table(lib, kern):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
    cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
    flag = "-gi" if os.environ.get("NCU_LINES_CALLSITE") else "-g"
    dis = subprocess.run(["nvdisasm", flag, "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
    tab, cur, on = {}, None, False
    for ln in dis.splitlines():
        if ln.startswith(".text."):
            on = kern in ln
            continue
        if not on:
            continue
        m = re.search(r'//## File "([^"]+)", line (\d+)(?: inlined at "([^"]+)", line (\d+))?', ln)
        if m:
            # NCU_LINES_CALLSITE=1: charge inlined helpers to their call site
            if m.group(3):
                cur = (os.path.basename(m.group(3)), int(m.group(4)))
            else:
                cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*)", ln)
        if m:
            tab[int(m.group(1), 16)] = (cur, m.group(2).strip())
    return tab


def main():
    rep, lib, kern = sys.argv[1:4]
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    rows = sass_rows(rep)
    base = int(rows[0][0], 16)
    tab = line_table(lib, kern)
    samp, inst = collections.Counter(), collections.Counter()
    # outlined wait loops (try_wait / nanosleep / branch back) carry the
    # helper's line only: charge them to the call site, i.e. the line of the
    # instruction just before the unconditional branch back into main code
    offs = [int(r[0], 16) - base for r in rows]
    site = {}
    blk = []
    for r, off in zip(rows, offs):
        txt = r[1].strip()
        blk.append(off)
        m = re.match(r"BRA\s+(0x[0-9a-f]+)", txt)
        if m or txt.startswith("EXIT"):
            if m:
                tgt = int(m.group(1), 16) - base
                if tgt < blk[0]:
                    prev = max((o for o in offs if o < tgt), default=None)
                    if prev is not None and prev in tab:
                        for o in blk:
                            if tab.get(o, ((None, 0), ""))[0][0] == "sm100.cuh" or "SYNCS" in tab.get(o, (0, ""))[1] \
                                    or "NANOSLEEP" in tab.get(o, (0, ""))[1]:
                                site[o] = tab[prev][0]
            blk = []
    for r, off in zip(rows, offs):
        src = tab.get(off, (("?", 0), ""))[0]
        if off in site:
            src = (site[off][0] + "(wait)", site[off][1])
        samp[src] += int(r[2] or 0)
        inst[src] += int(r[5] or 0)
    ts, ti = sum(samp.values()), sum(inst.values())
    print(f"samples {ts}  warp-instructions {ti}")
    print(f"{'file:line':32s} {'samples%':>8s} {'instr%':>7s}")
    for src, v in samp.most_common(top):
        print(f"{src[0]}:{src[1]:<18d} {100 * v / ts:8.2f} {100 * inst[src] / ti:7.2f}")


if __name__ == "__main__":
    main()
