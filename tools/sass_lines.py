"""Static SASS view of one kernel with source lines (no GPU needed).

  python tools/sass_lines.py LIB.so KERNEL_SUBSTR FILE LINE_LO LINE_HI
prints the SASS instructions whose innermost source line lies in
[LINE_LO, LINE_HI] of FILE (basename), in address order, so the hot loops'
instruction counts can be checked after every edit (-lineinfo build).
"""
import os
import re
import subprocess
import sys
import tempfile


def main():
    lib, kern, fname, lo, hi = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4]), int(sys.argv[5])
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
    cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
    dis = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
    cur, on, n = None, False, 0
    for ln in dis.splitlines():
        if ln.startswith(".text."):
            on = kern in ln
            continue
        if not on:
            continue
        m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
        if m and cur and cur[0] == fname and lo <= cur[1] <= hi:
            print(f"{m.group(1)} L{cur[1]:<5d} {m.group(2)}")
            n += 1
    print("instructions:", n)


if __name__ == "__main__":
    main()
